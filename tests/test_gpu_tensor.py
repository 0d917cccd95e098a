"""GPU parity of the tcgen05 3xTF32 contraction executor (engine=TENSOR) vs the fp64 oracle."""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu
E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")
TENSOR = 2


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(device="cuda", dtype=torch.float32)


def host(t):
    torch.cuda.synchronize()
    return t.double().cpu().numpy()


TILES = [(16, 1024, 16), (16, 128, 8), (32, 512, 16), (16, 256, 32), (48, 256, 8), (64, 128, 16)]


def test_tc_inapplicable_tile_is_reported_not_faked(cuda_device):
    # (48, 384): 2 M-blocks per converter warp x 48 columns > the 64 fp32 chunk sums per thread
    d = E.desc_builtin("gemm", (64, 384, 64)); d.set_exec(50, TENSOR)
    with pytest.raises(E.EatssError) as ei:
        E.run(d, (48, 384, 8), [dev(np.zeros((64, 384))), dev(np.zeros((64, 64))), dev(np.zeros((64, 384)))])
    assert ei.value.status == -5  # EATSS_E_UNSUPPORTED


@pytest.mark.parametrize("tiles", TILES)
def test_tc_gemm_small_int_bit_exact(cuda_device, tiles):
    ni, nj, nk = 300, 1100, 204  # ragged i/j tiles and a ragged last k stage (204 = 25*8+4)
    A = synth.small_int((ni, nk), 10); B = synth.small_int((nk, nj), 11); C = synth.small_int((ni, nj), 12)
    ref = O.gemm(1.0, 1.0, C, A, B)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 1.0); d.set_exec(50, TENSOR)
    Cd = dev(C)
    E.run(d, tiles, [Cd, dev(A), dev(B)])
    assert np.array_equal(host(Cd), ref)


@pytest.mark.parametrize("tiles", TILES)
def test_tc_gemm_random_tolerance(cuda_device, tiles):
    ni, nj, nk = 260, 516, 1000
    A = synth.uniform((ni, nk), 20); B = synth.uniform((nk, nj), 21); C = synth.uniform((ni, nj), 22)
    ref = O.gemm(1.5, 1.2, C, A, B)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR)
    Cd = dev(C)
    E.run(d, tiles, [Cd, dev(A), dev(B)])
    assert O.normwise_rel_err(host(Cd), ref) <= 1e-5


def test_tc_gemm_full_size_sampled(cuda_device):
    """The narrow-tile TS engine at N=4000: the truncating tf32 accumulation is drained into fp32
    registers every 128 k (tc_gemm.cu), which keeps the 3xTF32 error at the fp32 level."""
    n = 4000
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR)
    A = synth.uniform((n, n), 4); B = synth.uniform((n, n), 5); C = synth.uniform((n, n), 6)
    Cd = dev(C)
    E.run(d, (16, 1024, 16), [Cd, dev(A), dev(B)])
    out = host(Cd)
    g = synth.rng(7)
    ii = g.integers(0, n, 2048); jj = g.integers(0, n, 2048)
    assert O.normwise_rel_err(out[ii, jj], O.gemm_entries(ii, jj, C, A, B, 1.5, 1.2)) <= 1e-5


def test_tc_2mm_3mm(cuda_device):
    ni, nj, nk, nl = 131, 260, 96, 300
    A = synth.uniform((ni, nk), 50); B = synth.uniform((nk, nj), 51)
    C = synth.uniform((nj, nl), 52); D = synth.uniform((ni, nl), 53)
    tmp_ref, D_ref = O.two_mm(1.5, 1.2, A, B, C, D)
    d = E.desc_builtin("2mm", (ni, nj, nk, nl)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR)
    tmp = torch.zeros((ni, nj), device="cuda"); Dd = dev(D)
    E.run(d, (16, 1024, 16), [tmp, dev(A), dev(B), dev(C), Dd])
    assert O.normwise_rel_err(host(tmp), tmp_ref) <= 1e-5 and O.normwise_rel_err(host(Dd), D_ref) <= 1e-5


# ---- MMA-legal tiles (Ti = 128): TMA + SS-UMMA GEMM (tc_mma.cu)
MMA_TILES = [(256, 256, 32), (128, 256, 32), (128, 128, 32), (128, 64, 8), (128, 192, 16), (128, 32, 32),
             (256, 96, 64), (128, 48, 16), (128, 208, 32), (256, 64, 8), (256, 160, 16), (128, 16, 64)]


@pytest.mark.parametrize("tiles", MMA_TILES)
def test_tcm_small_int_bit_exact(cuda_device, tiles):
    ni, nj, nk = 300, 1100, 204  # ragged everywhere: TMA zero-fill at the i/j/k edges
    A = synth.small_int((ni, nk), 10); B = synth.small_int((nk, nj), 11); C = synth.small_int((ni, nj), 12)
    ref = O.gemm(1.0, 1.0, C, A, B)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 1.0); d.set_exec(50, TENSOR)
    Cd = dev(C)
    E.run(d, tiles, [Cd, dev(A), dev(B)])
    assert np.array_equal(host(Cd), ref)


@pytest.mark.parametrize("tiles", MMA_TILES[:3])
def test_tcm_random_tolerance(cuda_device, tiles):
    ni, nj, nk = 260, 516, 1000
    A = synth.uniform((ni, nk), 20); B = synth.uniform((nk, nj), 21); C = synth.uniform((ni, nj), 22)
    ref = O.gemm(1.5, 1.2, C, A, B)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR)
    Cd = dev(C)
    E.run(d, tiles, [Cd, dev(A), dev(B)])
    assert O.normwise_rel_err(host(Cd), ref) <= 1e-5


def test_tcm_full_size_sampled(cuda_device):
    n = 4000
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR)
    A = synth.uniform((n, n), 4); B = synth.uniform((n, n), 5); C = synth.uniform((n, n), 6)
    Cd = dev(C)
    E.run(d, (256, 256, 32), [Cd, dev(A), dev(B)])
    out = host(Cd)
    g = synth.rng(7)
    ii = g.integers(0, n, 2048); jj = g.integers(0, n, 2048)
    assert O.normwise_rel_err(out[ii, jj], O.gemm_entries(ii, jj, C, A, B, 1.5, 1.2)) <= 1e-5


# ---- syrk on the tensor pipe: B(k, j) = A(j, k) is K-major (same operand layout as A)
SYRK_TILES = [(256, 256, 32), (128, 256, 32), (128, 224, 16), (128, 96, 32), (128, 32, 8), (256, 48, 32),
              (256, 80, 64), (128, 16, 16)]


@pytest.mark.parametrize("tiles", SYRK_TILES)
def test_tcm_syrk_small_int_exact_and_random(cuda_device, tiles):
    ni, nj = 403, 157  # odd pitch: operands are re-pitched to 16-byte rows for TMA
    Ai = synth.small_int((ni, nj), 72); Ci = synth.small_int((ni, ni), 73)
    d = E.desc_builtin("syrk", (ni, nj)); d.set_scalars(1.0, 1.0); d.set_exec(50, TENSOR)
    Cd = dev(Ci)
    E.run(d, tiles, [Cd, dev(Ai)])
    assert np.array_equal(host(Cd), O.syrk(1.0, 1.0, Ci, Ai))
    A = synth.uniform((ni, nj), 70); C = synth.uniform((ni, ni), 71)
    d.set_scalars(1.5, 1.2)
    Cd = dev(C)
    E.run(d, tiles, [Cd, dev(A)])
    assert O.normwise_rel_err(host(Cd), O.syrk(1.5, 1.2, C, A)) <= 1e-5


def test_tcm_syrk_row_block(cuda_device):
    # rows [r0, r0 + rows) of C only (the multi-GPU shard form): A operand is a row block of B
    ni, nj, r0, rows = 300, 200, 77, 150
    A = synth.uniform((ni, nj), 80); C = synth.uniform((ni, ni), 81)
    ref = O.syrk(1.5, 1.2, C, A)
    d = E.desc_builtin("syrk", (ni, nj, r0, rows)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR)
    Cb = dev(C[r0:r0 + rows])
    E.run(d, (128, 128, 32), [Cb, dev(A)])
    assert O.normwise_rel_err(host(Cb), ref[r0:r0 + rows]) <= 1e-5


def test_tcm_syrk_full_size_sampled(cuda_device):
    n = 4000
    A = synth.uniform((n, n), 8); C = synth.uniform((n, n), 9)
    d = E.desc_builtin("syrk", (n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR)
    Cd = dev(C)
    E.run(d, (256, 256, 32), [Cd, dev(A)])
    out = host(Cd)
    g = synth.rng(10)
    ii = g.integers(0, n, 2048); jj = g.integers(0, n, 2048)
    want = O.gemm_entries(ii, jj, C, A, np.ascontiguousarray(A.T), 1.5, 1.2)
    assert O.normwise_rel_err(out[ii, jj], want) <= 1e-5


@pytest.mark.parametrize("splitk", ["0", "1"])
def test_tcm_tail_split_on_and_off(cuda_device, monkeypatch, splitk):
    # 600 x 1300 with (128, 256): 3 pair-rows x 6 column tiles = 18 tiles < the clusters of one
    # wave, so with split-k on every tile is split along k (atomics on a beta-prescaled C)
    monkeypatch.setenv("EATSS_TCM_SPLITK", splitk)
    ni, nj, nk = 600, 1300, 2000
    A = synth.small_int((ni, nk), 30); B = synth.small_int((nk, nj), 31); C = synth.small_int((ni, nj), 32)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 2.0); d.set_exec(50, TENSOR)
    Cd = dev(C)
    E.run(d, (256, 256, 32), [Cd, dev(A), dev(B)])
    assert np.array_equal(host(Cd), O.gemm(1.0, 2.0, C, A, B))


@pytest.mark.parametrize("tiles", [(256, 256, 32), (128, 256, 32), (128, 160, 32), (256, 96, 16)])
def test_tcm_2mm_3mm(cuda_device, tiles):
    ni, nj, nk, nl, nm = 331, 260, 296, 300, 140
    A = synth.uniform((ni, nk), 50); B = synth.uniform((nk, nj), 51)
    C = synth.uniform((nj, nl), 52); D = synth.uniform((ni, nl), 53)
    tmp_ref, D_ref = O.two_mm(1.5, 1.2, A, B, C, D)
    d = E.desc_builtin("2mm", (ni, nj, nk, nl)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR)
    tmp = torch.full((ni, nj), float("nan"), device="cuda"); Dd = dev(D)  # init_zero: never read
    E.run(d, tiles, [tmp, dev(A), dev(B), dev(C), Dd])
    assert O.normwise_rel_err(host(tmp), tmp_ref) <= 1e-5 and O.normwise_rel_err(host(Dd), D_ref) <= 1e-5
    C3 = synth.uniform((nj, nm), 54); D3 = synth.uniform((nm, nl), 55)
    E_ref, F_ref, G_ref = O.three_mm(A, B, C3, D3)
    d = E.desc_builtin("3mm", (ni, nj, nk, nl, nm)); d.set_exec(50, TENSOR)
    Eb, Fb, Gb = (torch.full(s, float("nan"), device="cuda") for s in ((ni, nj), (nj, nl), (ni, nl)))
    E.run(d, tiles, [Eb, dev(A), dev(B), Fb, dev(C3), dev(D3), Gb])
    for got, want in ((Eb, E_ref), (Fb, F_ref), (Gb, G_ref)):
        assert O.normwise_rel_err(host(got), want) <= 1e-5


@pytest.mark.parametrize("tiles", [(256, 256, 32), (128, 96, 32), (128, 48, 8)])
def test_tcm_split_exact_for_22_bit_values(cuda_device, tiles):
    # hi + lo reproduces every fp32 value with <= 22 significant bits exactly, whichever split
    # mode is active (rna hi, or the raw operand read by the truncating tensor core): A @ I == A
    n = 300
    g = synth.rng(90)
    A = (g.integers(2 ** 21, 2 ** 22, (n, n)) * g.choice([-1.0, 1.0], (n, n))) * 2.0 ** -21
    A = A * 2.0 ** g.integers(-6, 6, (n, n))
    A = A.astype(np.float32).astype(np.float64)
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.0, 0.0); d.set_exec(50, TENSOR)
    Cd = torch.zeros((n, n), device="cuda")
    E.run(d, tiles, [Cd, dev(A), dev(np.eye(n))])
    assert np.array_equal(host(Cd), A)


def test_kernel_timing_and_launch_count(cuda_device):
    # exec.time_kernels: events around the GEMM launch alone; launches_per_run counts the fused
    # prep launch (operand splits of A and B -- syrk shares one -- and the split-k tail pre-pass
    # when beta != 1) and the GEMM
    n = 2500
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(1.5, 1.2); d.set_exec(50, TENSOR, time_kernels=1)
    bufs = [torch.rand(n, n, device="cuda") for _ in range(3)]
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    E.run(d, (256, 256, 32), bufs)
    s.record(); E.run(d, (256, 256, 32), bufs); e.record()
    torch.cuda.synchronize()
    (k,) = E.last_kernel_ms(d)
    assert 0 < k < s.elapsed_time(e)
    # 2500/256 -> 10 pair-rows x 10 column tiles = 100 tiles on 74 clusters: the 26-tile tail is
    # split along k (pre-pass needed for beta != 1, run inside the prep launch)
    assert E.launches_per_run(d, (256, 256, 32)) == 2
    d.set_scalars(1.5, 1.0)
    assert E.launches_per_run(d, (256, 256, 32)) == 2
    ds = E.desc_builtin("syrk", (n, n)); ds.set_exec(50, TENSOR)
    assert E.launches_per_run(ds, (256, 256, 32)) == 2
    d2 = E.desc_builtin("gemm", (n, n, n))
    with pytest.raises(E.EatssError):
        E.last_kernel_ms(d2)


# ---- ccsd_t_d1 on the tensor pipe (ccsd_tc.cu): tile (1, 1, Th1, Tp6, Tp5, Tp4, >= H7)
CCSD_TC = [((16,) * 7, (1, 1, 1, 16, 8, 16, 16)), ((16,) * 7, (1, 1, 2, 16, 4, 16, 16)),
           ((16,) * 7, (1, 1, 1, 16, 2, 16, 16)),
           ((3, 5, 6, 20, 7, 12, 20), (1, 1, 2, 16, 3, 12, 20)),   # ragged h1/p5/p6 tiles, h7 pad
           ((2, 3, 4, 32, 4, 8, 48), (1, 1, 2, 32, 4, 8, 48)),    # two k-blocks (H7 = 48)
           ((2, 2, 3, 160, 2, 16, 16), (1, 1, 1, 160, 2, 16, 16)),  # N = 160: one TMEM accumulator
           ((16,) * 7, (1, 2, 1, 16, 4, 16, 16)),                  # Th2 = 2: N = (h2, p6) = 32
           ((2, 3, 4, 32, 4, 8, 48), (1, 2, 2, 32, 4, 8, 48)),      # ragged h2 tile (H2 = 3), two k-blocks
           ((3, 5, 3, 16, 5, 12, 20), (1, 4, 2, 16, 3, 12, 20))]   # N = 64, ragged h1/p5, h7 pad


@pytest.mark.parametrize("dims,tiles", CCSD_TC)
def test_ccsd_tc(cuda_device, dims, tiles):
    H3, H2, H1, P6, P5, P4, H7 = dims
    d = E.desc_builtin("ccsd_t_d1", dims); d.set_exec(50, TENSOR)
    t3i = synth.small_int((H3, H2, H1, P6, P5, P4), 103)
    t2i = synth.small_int((H7, P4, P5, H1), 104); v2i = synth.small_int((H3, H2, P6, H7), 105)
    t3d = dev(t3i)
    E.run(d, tiles, [t3d, dev(t2i), dev(v2i)])
    assert np.array_equal(host(t3d), O.ccsd_t_d1(t3i, t2i, v2i))
    t3 = synth.uniform(t3i.shape, 100); t2 = synth.uniform(t2i.shape, 101); v2 = synth.uniform(v2i.shape, 102)
    t3d = dev(t3)
    E.run(d, tiles, [t3d, dev(t2), dev(v2)])
    assert O.normwise_rel_err(host(t3d), O.ccsd_t_d1(t3, t2, v2)) <= 1e-5


def test_ccsd_tc_rejects_non_mma_tiles(cuda_device):
    d = E.desc_builtin("ccsd_t_d1", (16,)); d.set_exec(50, TENSOR)
    bufs = [torch.zeros(d.buffer_elems(i), device="cuda") for i in range(3)]
    for tiles in [(4, 4, 4, 4, 4, 32, 4), (1, 1, 1, 16, 16, 16, 16), (1, 1, 1, 8, 8, 16, 16), (1, 1, 1, 16, 8, 16, 8)]:
        with pytest.raises(E.EatssError) as ei:
            E.run(d, tiles, bufs)
        assert ei.value.status == -5


CCSD_TC_TILE48 = (1, 2, 2, 48, 1, 48, 48)  # the other tied optimum of reading T4


def test_ccsd_tc_model_tiles_run_exact(cuda_device):
    """Reading T4 (tensor mode of eatss_select_tiles for the 6-D contraction) picks executable tiles:
    small-integer inputs give the oracle's exact result at several shapes."""
    gpu = E.gpu_params_query(0)
    for dims in [(16,) * 7, (3, 5, 6, 20, 7, 12, 20), (2, 3, 4, 32, 4, 8, 48), (24,) * 7]:
        H3, H2, H1, P6, P5, P4, H7 = dims
        d = E.desc_builtin("ccsd_t_d1", dims); d.set_exec(50, TENSOR)
        tiles, _ = E.select_tiles(d, gpu, 50, 4, mode=2)
        t3i = synth.small_int((H3, H2, H1, P6, P5, P4), 113)
        t2i = synth.small_int((H7, P4, P5, H1), 114); v2i = synth.small_int((H3, H2, P6, H7), 115)
        t3d = dev(t3i)
        E.run(d, tiles, [t3d, dev(t2i), dev(v2i)])
        assert np.array_equal(host(t3d), O.ccsd_t_d1(t3i, t2i, v2i)), (dims, tiles)


@pytest.mark.parametrize("source", ["model", "hand"])
def test_ccsd_tc_full_size_dims48_sampled(cuda_device, source):
    n = 48
    d = E.desc_builtin("ccsd_t_d1", (n,)); d.set_exec(50, TENSOR)
    tiles = E.select_tiles(d, E.gpu_params_query(0), 50, 4, mode=2)[0] if source == "model" else CCSD_TC_TILE48
    if source == "model":
        assert tiles == (1, 2, 1, 48, 2, 48, 48)  # tests/test_oracle_model.py::test_tensor_mode_6d_hand_checked
    t2 = synth.uniform((n, n, n, n), 110); v2 = synth.uniform((n, n, n, n), 111)
    t3d = torch.zeros(n ** 6, dtype=torch.float32, device="cuda")
    E.run(d, tiles, [t3d, dev(t2), dev(v2)])
    g = synth.rng(112)
    idx = np.concatenate([g.integers(0, n ** 6, 100000), np.arange(n ** 4) + 7 * n ** 5 + 3 * n ** 4])
    got = t3d[torch.from_numpy(idx).cuda()].double().cpu().numpy()
    ref = O.ccsd_t_d1_entries((n,) * 7, idx, np.zeros(len(idx)), t2, v2)
    assert O.normwise_rel_err(got, ref) <= 1e-5
    del t3d
    torch.cuda.empty_cache()


# ---- the whole tensor-engine tile space: Ti in {128, 256}, Tj in 16..256 step 16,
# Tk in {8, 16, 32, 64}; every executable tile exact on small integers (gemm: MN-major B; syrk: K-major)
def _space():
    return [(ti, tj, tk) for ti in (128, 256) for tj in range(16, 257, 16) for tk in (8, 16, 32, 64)]


@pytest.fixture(scope="module")
def space_inputs():
    ni, nj, nk = 300, 1100, 204
    A = synth.small_int((ni, nk), 10); B = synth.small_int((nk, nj), 11); C = synth.small_int((ni, nj), 12)
    As = synth.small_int((ni, nk), 13); Cs = synth.small_int((ni, ni), 14)
    return (ni, nj, nk), (A, B, C, O.gemm(1.0, 1.0, C, A, B)), (As, Cs, O.syrk(1.0, 1.0, Cs, As))


def test_tcm_whole_tile_space_exact(cuda_device, space_inputs):
    (ni, nj, nk), (A, B, C, ref), (As, Cs, refs) = space_inputs
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 1.0); d.set_exec(50, TENSOR)
    ds = E.desc_builtin("syrk", (ni, nk)); ds.set_scalars(1.0, 1.0); ds.set_exec(50, TENSOR)
    Ad, Bd, Asd = dev(A), dev(B), dev(As)
    ran = {"gemm": 0, "syrk": 0}
    for t in _space():
        for name, dd, mk, r in (("gemm", d, lambda: [dev(C), Ad, Bd], ref), ("syrk", ds, lambda: [dev(Cs), Asd], refs)):
            b = mk()
            try:
                E.run(dd, t, b)
            except E.EatssError as err:
                assert err.status == -5, (name, t)  # EATSS_E_UNSUPPORTED: shared memory / legal N only
                ti, tj, tk = t
                assert (name == "gemm" and ti == 256 and (tj // 2) % 16) or tk == 64, (name, t)
                continue
            assert np.array_equal(host(b[0]), r), (name, t)
            ran[name] += 1
    assert ran["gemm"] >= 80 and ran["syrk"] >= 80, ran


def test_tcm_model_space_is_executable(cuda_device):
    """Every tile reading T declares feasible (tensor mode of eatss_select_tiles) is one
    the executor accepts: the model's T3 constraints are the executor's legality + shared memory."""
    from oracle import model as M
    doms = M.tensor_domains(M.gemm())
    import itertools
    feas = [t for t in itertools.product(*doms)
            if M.evaluate_tensor(M.gemm(), M.B200, M.Opts(50, 16, 2), [np.array([v]) for v in t])[0][0]]
    assert len(feas) == 36
    n = 512
    d = E.desc_builtin("gemm", (n, n, n)); d.set_exec(50, TENSOR)
    bufs = [torch.zeros((n, n), device="cuda") for _ in range(3)]
    for t in feas:
        E.run(d, t, bufs)
    torch.cuda.synchronize()

"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Bars (north star): fp32 normwise relative error <= 1e-5, fp64 <= 1e-12, integer /
index work bit-exact.  Small-integer inputs make every fp32 partial sum exact
(|sum| < 2^24), so those runs must equal the oracle bit for bit for ANY tiling.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu

E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")

TOL32, TOL64 = 1e-5, 1e-12


def dev(x, dtype=torch.float32):
    return torch.from_numpy(np.ascontiguousarray(x)).to(device="cuda", dtype=dtype)


def host(t):
    torch.cuda.synchronize()
    return t.double().cpu().numpy()


def run(d, tiles, bufs):
    E.run(d, tiles, bufs)
    torch.cuda.synchronize()


# ------------------------------------------------------------------ gemm
def test_config1_gemm_256_tile32(cuda_device):
    n = 256
    A = synth.uniform((n, n), 0); B = synth.uniform((n, n), 1); C = synth.uniform((n, n), 2)
    a, b = np.float32(1.5), np.float32(1.2)
    ref = O.gemm(float(a), float(b), C, A, B)
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(float(a), float(b))
    Cd = dev(C)
    run(d, (32, 32, 32), [Cd, dev(A), dev(B)])
    assert O.normwise_rel_err(host(Cd), ref) <= TOL32


GEMM_TILES = [(32, 32, 32), (16, 1024, 16), (4, 4, 4), (1024, 1024, 1024), (24, 96, 48), (7, 13, 5),
              (128, 8, 3), (64, 1024, 1), (1, 1, 64), (512, 384, 16)]


@pytest.mark.parametrize("tiles", GEMM_TILES)
def test_gemm_small_int_bit_exact_ragged(cuda_device, tiles):
    ni, nj, nk = 301, 267, 259  # ragged in every dimension, not multiples of 4
    A = synth.small_int((ni, nk), 10); B = synth.small_int((nk, nj), 11); C = synth.small_int((ni, nj), 12)
    ref = O.gemm(1.0, 1.0, C, A, B)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 1.0)
    Cd = dev(C)
    run(d, tiles, [Cd, dev(A), dev(B)])
    assert np.array_equal(host(Cd), ref)


@pytest.mark.parametrize("tiles", GEMM_TILES)
def test_gemm_vec4_path_random(cuda_device, tiles):
    ni, nj, nk = 260, 516, 132  # multiples of 4: 16-byte vector path
    A = synth.uniform((ni, nk), 20); B = synth.uniform((nk, nj), 21); C = synth.uniform((ni, nj), 22)
    ref = O.gemm(1.5, 1.2, C, A, B)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.5, 1.2)
    Cd = dev(C)
    run(d, tiles, [Cd, dev(A), dev(B)])
    assert O.normwise_rel_err(host(Cd), ref) <= TOL32


def test_gemm_identity_and_rank1(cuda_device):
    n = 192
    A = synth.small_int((n, n), 30); C = synth.small_int((n, n), 31)
    d = E.desc_builtin("gemm", (n, n, n)); d.set_scalars(2.0, 0.5)
    Cd = dev(C)
    run(d, (16, 64, 16), [Cd, dev(A), dev(np.eye(n, dtype=np.float32))])
    assert np.array_equal(host(Cd), 0.5 * C.astype(np.float64) + 2.0 * A)
    g = synth.rng(32)
    u, v, w, x = (g.integers(-3, 4, n) for _ in range(4))
    d.set_scalars(1.0, 0.0)
    Cd = dev(np.zeros((n, n), np.float32))
    run(d, (32, 128, 8), [Cd, dev(np.outer(u, v)), dev(np.outer(w, x))])
    assert np.array_equal(host(Cd), float(v @ w) * np.outer(u, x))


def test_gemm_f64_tolerance(cuda_device):
    ni, nj, nk = 130, 97, 211
    A = synth.uniform((ni, nk), 40, dtype=np.float64); B = synth.uniform((nk, nj), 41, dtype=np.float64)
    C = synth.uniform((ni, nj), 42, dtype=np.float64)
    ref = O.gemm(1.5, 1.2, C, A, B)
    d = E.desc_builtin("gemm", (ni, nj, nk), "f64"); d.set_scalars(1.5, 1.2)
    for tiles in [(16, 512, 16), (32, 32, 32), (5, 7, 300)]:
        Cd = dev(C, torch.float64)
        run(d, tiles, [Cd, dev(A, torch.float64), dev(B, torch.float64)])
        assert O.normwise_rel_err(host(Cd), ref) <= TOL64


@pytest.mark.parametrize("tiles,shape", [((16, 1024, 16), (70, 1100, 33)), ((32, 32, 32), (65, 33, 31)),
                                         ((5, 7, 3), (23, 19, 11)), ((1024, 1024, 4), (40, 1030, 9)),
                                         ((48, 8, 1024), (100, 30, 20))])
def test_coverage_every_point_exactly_once(cuda_device, tiles, shape):
    ni, nj, nk = shape
    d = E.desc_builtin("gemm", shape)
    counts = torch.zeros(ni * nj * nk, dtype=torch.int32, device="cuda")
    E.coverage(d, 0, tiles, counts)
    c = counts.cpu().numpy()
    assert c.min() == 1 and c.max() == 1


def test_gemm_full_size_eatss_tile_sampled(cuda_device):
    """gemm N=4000 with the EATSS tile, in the launch configuration bench.py times."""
    n = 4000
    d = E.desc_builtin("gemm", (n, n, n))
    tiles, _ = E.select_tiles(d, E.gpu_params_query(0), 50, 16)
    # 1000 tiles on 2 x 148 resident CTAs: the last wave's tiles are split along k (tail pre-pass +
    # atomic k-parts), which these samples reach (tail rows >= 3552 get their own 512 samples)
    d.set_exec(50, 1)
    assert E.launches_per_run(d, tiles) == 2
    g = synth.rng(7)
    ii = np.concatenate([g.integers(0, n, 2048), g.integers(3552, n, 512)])
    jj = g.integers(0, n, len(ii))
    # small-int pass: every output must be exact (checked on 2048 sampled entries)
    A = synth.small_int((n, n), 1); B = synth.small_int((n, n), 2); C = synth.small_int((n, n), 3)
    d.set_scalars(1.0, 1.0)
    Cd = dev(C)
    run(d, tiles, [Cd, dev(A), dev(B)])
    out = host(Cd)
    assert np.array_equal(out[ii, jj], O.gemm_entries(ii, jj, C, A, B, 1.0, 1.0))
    assert np.array_equal(out, np.round(out))  # property at every entry: integers stay integers
    # random signed pass: sampled normwise error
    A = synth.uniform((n, n), 4); B = synth.uniform((n, n), 5); C = synth.uniform((n, n), 6)
    d.set_scalars(1.5, 1.2)
    Cd = dev(C)
    run(d, tiles, [Cd, dev(A), dev(B)])
    out = host(Cd)
    ref = O.gemm_entries(ii, jj, C, A, B, 1.5, 1.2)
    assert O.normwise_rel_err(out[ii, jj], ref) <= TOL32


# ------------------------------------------------------------- 2mm / 3mm / syrk
@pytest.mark.parametrize("tiles", [(16, 1024, 16), (32, 32, 32), (9, 40, 7)])
def test_2mm(cuda_device, tiles):
    ni, nj, nk, nl = 131, 145, 99, 120
    A = synth.uniform((ni, nk), 50); B = synth.uniform((nk, nj), 51)
    C = synth.uniform((nj, nl), 52); D = synth.uniform((ni, nl), 53)
    tmp_ref, D_ref = O.two_mm(1.5, 1.2, A, B, C, D)
    d = E.desc_builtin("2mm", (ni, nj, nk, nl)); d.set_scalars(1.5, 1.2)
    tmp = torch.full((ni, nj), float("nan"), device="cuda"); Dd = dev(D)
    run(d, tiles, [tmp, dev(A), dev(B), dev(C), Dd])
    assert O.normwise_rel_err(host(tmp), tmp_ref) <= TOL32
    assert O.normwise_rel_err(host(Dd), D_ref) <= TOL32


def test_2mm_small_int_exact(cuda_device):
    ni, nj, nk, nl = 200, 150, 180, 170
    A = synth.small_int((ni, nk), 54, -1, 1); B = synth.small_int((nk, nj), 55, -1, 1)
    C = synth.small_int((nj, nl), 56, -1, 1); D = synth.small_int((ni, nl), 57, -1, 1)
    tmp_ref, D_ref = O.two_mm(1.0, 1.0, A, B, C, D)
    d = E.desc_builtin("2mm", (ni, nj, nk, nl)); d.set_scalars(1.0, 1.0)
    tmp = torch.zeros((ni, nj), device="cuda"); Dd = dev(D)
    run(d, (16, 128, 16), [tmp, dev(A), dev(B), dev(C), Dd])
    assert np.array_equal(host(tmp), tmp_ref) and np.array_equal(host(Dd), D_ref)


@pytest.mark.parametrize("tiles", [(16, 1024, 16), (64, 64, 8)])
def test_3mm_and_run_nest(cuda_device, tiles):
    ni, nj, nk, nl, nm = 90, 110, 70, 130, 60
    A = synth.sparse_ternary((ni, nk), 60); B = synth.sparse_ternary((nk, nj), 61)
    C = synth.sparse_ternary((nj, nm), 62); D = synth.sparse_ternary((nm, nl), 63)
    Er, Fr, Gr = O.three_mm(A, B, C, D)
    assert max(abs(Er).max(), abs(Fr).max(), abs(Gr).max()) < 2 ** 24  # exactness certificate
    d = E.desc_builtin("3mm", (ni, nj, nk, nl, nm))
    bufs = [torch.full((ni, nj), float("nan"), device="cuda"), dev(A), dev(B),
            torch.full((nj, nl), float("nan"), device="cuda"), dev(C), dev(D),
            torch.full((ni, nl), float("nan"), device="cuda")]
    run(d, tiles, bufs)
    assert np.array_equal(host(bufs[0]), Er) and np.array_equal(host(bufs[3]), Fr)
    assert np.array_equal(host(bufs[6]), Gr)
    for t in (bufs[0], bufs[3], bufs[6]):
        t.fill_(float("nan"))
    for nest in range(3):
        E.run_nest(d, nest, tiles, bufs)
    torch.cuda.synchronize()
    assert np.array_equal(host(bufs[6]), Gr)


@pytest.mark.parametrize("tiles", [(16, 1024, 16), (32, 32, 32), (11, 5, 64), (256, 256, 256)])
def test_syrk(cuda_device, tiles):
    ni, nj = 203, 157
    A = synth.uniform((ni, nj), 70); C = synth.uniform((ni, ni), 71)
    ref = O.syrk(1.5, 1.2, C, A)
    d = E.desc_builtin("syrk", (ni, nj)); d.set_scalars(1.5, 1.2)
    Cd = dev(C)
    run(d, tiles, [Cd, dev(A)])
    assert O.normwise_rel_err(host(Cd), ref) <= TOL32
    Ai = synth.small_int((ni, nj), 72); Ci = synth.small_int((ni, ni), 73)
    d.set_scalars(1.0, 1.0)
    Cd = dev(Ci)
    run(d, tiles, [Cd, dev(Ai)])
    assert np.array_equal(host(Cd), O.syrk(1.0, 1.0, Ci, Ai))


# ------------------------------------------------------------------ stencils
@pytest.mark.parametrize("n,tiles,T", [(130, (16, 1024), 21), (128, (32, 32), 20), (67, (5, 12), 7),
                                       (200, (1024, 1024), 1), (96, (16, 64), 0)])
def test_jacobi2d(cuda_device, n, tiles, T):
    A, B = synth.polybench_jacobi2d(n)
    Ar, Br = O.jacobi2d(A, B, T)
    d = E.desc_builtin("jacobi-2d", (n,), tsteps=T)
    Ad, Bd = dev(A), dev(B)
    run(d, tiles, [Ad, Bd])
    assert O.normwise_rel_err(host(Ad), Ar) <= TOL32 and O.normwise_rel_err(host(Bd), Br) <= TOL32
    # boundaries bit-exact untouched
    for X, X0 in ((host(Ad), A), (host(Bd), B)):
        assert np.array_equal(X[0], X0[0]) and np.array_equal(X[-1], X0[-1])
        assert np.array_equal(X[:, 0], X0[:, 0]) and np.array_equal(X[:, -1], X0[:, -1])


def test_jacobi2d_random_and_graph_replay(cuda_device):
    n, T = 256, 30
    A = synth.uniform((n, n), 80); B = synth.uniform((n, n), 81)
    Ar, Br = O.jacobi2d(A, B, T)
    d = E.desc_builtin("jacobi-2d", (n,), tsteps=T)
    for _ in range(2):  # second call replays the cached CUDA graph
        Ad, Bd = dev(A), dev(B)
        run(d, (16, 1024), [Ad, Bd])
    assert O.normwise_rel_err(host(Ad), Ar) <= TOL32 and O.normwise_rel_err(host(Bd), Br) <= TOL32


def test_jacobi2d_linear_field_exact_full_size(cuda_device):
    n, T = 4000, 5
    A = synth.linear_field((n, n), (3, -2), 7); B = synth.linear_field((n, n), (1, 5), -4)
    d = E.desc_builtin("jacobi-2d", (n,), tsteps=T)
    Ad, Bd = dev(A), dev(B)
    run(d, (16, 1024), [Ad, Bd])
    assert np.array_equal(host(Ad), A)
    Bh = host(Bd)
    assert np.array_equal(Bh[1:-1, 1:-1], A[1:-1, 1:-1]) and np.array_equal(Bh[0], B[0])


@pytest.mark.parametrize("n,tiles,T", [(40, (16, 16, 32), 6), (34, (4, 24, 112), 5), (23, (3, 5, 7), 3),
                                       (120, (16, 16, 32), 2)])
def test_heat3d(cuda_device, n, tiles, T):
    A, B = synth.polybench_heat3d(n)
    A = A + synth.uniform(A.shape, 90) * 0.1  # break near-linearity of the P init
    Ar, Br = O.heat3d(A, B, T)
    d = E.desc_builtin("heat-3d", (n,), tsteps=T)
    Ad, Bd = dev(A), dev(B)
    run(d, tiles, [Ad, Bd])
    assert O.normwise_rel_err(host(Ad), Ar) <= TOL32 and O.normwise_rel_err(host(Bd), Br) <= TOL32


@pytest.mark.parametrize("kind,n,T", [("jacobi-2d", 4000, 500), ("heat-3d", 120, 500)])
def test_stencil_baseline_config_full(cuda_device, kind, n, T):
    """BASELINE config 4 at full size and full time-step count, with the model-selected tile (the
    tile bench.py times), random U[-1,1) fields, every output element compared."""
    d = E.desc_builtin(kind, (n,), tsteps=T)
    tiles, _ = E.select_tiles(d, E.gpu_params_query(0), 50, 16)
    shape = (n, n) if kind == "jacobi-2d" else (n, n, n)
    A = synth.uniform(shape, 95); B = synth.uniform(shape, 96)
    Ar, Br = (O.jacobi2d if kind == "jacobi-2d" else O.heat3d)(A, B, T)
    Ad, Bd = dev(A), dev(B)
    run(d, tiles, [Ad, Bd])
    assert O.normwise_rel_err(host(Ad), Ar) <= TOL32 and O.normwise_rel_err(host(Bd), Br) <= TOL32


def test_heat3d_linear_field_exact(cuda_device):
    n = 120
    A = synth.linear_field((n, n, n), (2, -3, 1), 5)
    d = E.desc_builtin("heat-3d", (n,), tsteps=10)
    Ad, Bd = dev(A), dev(A.copy())
    run(d, (16, 16, 32), [Ad, Bd])
    assert np.array_equal(host(Ad), A) and np.array_equal(host(Bd), A)


@pytest.mark.parametrize("kind,n,tiles", [("jacobi-2d", 67, (16, 1024)), ("jacobi-2d", 50, (5, 7)),
                                          ("heat-3d", 21, (4, 8, 16)), ("heat-3d", 30, (16, 16, 32))])
def test_stencil_coverage(cuda_device, kind, n, tiles):
    d = E.desc_builtin(kind, (n,), tsteps=1)
    dims = 2 if kind == "jacobi-2d" else 3
    counts = torch.zeros(n ** dims, dtype=torch.int32, device="cuda")
    E.coverage(d, 0, tiles, counts)
    c = counts.cpu().numpy().reshape((n,) * dims)
    inner = c[(slice(1, -1),) * dims]
    assert inner.min() == 1 and inner.max() == 1 and c.sum() == (n - 2) ** dims


# ------------------------------------------------------------------ ccsd_t_d1
@pytest.mark.parametrize("dims,tiles", [((16,) * 7, (4, 4, 4, 4, 4, 32, 4)), ((16,) * 7, (4, 8, 4, 4, 4, 16, 4)),
                                        ((5, 6, 7, 9, 10, 33, 11), (4, 4, 4, 4, 4, 32, 4)),
                                        ((5, 6, 7, 9, 10, 33, 11), (2, 3, 5, 4, 7, 8, 5)),
                                        ((8,) * 7, (8, 8, 8, 8, 8, 8, 8))])
def test_ccsd_t_d1(cuda_device, dims, tiles):
    H3, H2, H1, P6, P5, P4, H7 = dims
    t3 = synth.uniform((H3, H2, H1, P6, P5, P4), 100)
    t2 = synth.uniform((H7, P4, P5, H1), 101); v2 = synth.uniform((H3, H2, P6, H7), 102)
    ref = O.ccsd_t_d1(t3, t2, v2)
    d = E.desc_builtin("ccsd_t_d1", dims)
    t3d = dev(t3)
    run(d, tiles, [t3d, dev(t2), dev(v2)])
    assert O.normwise_rel_err(host(t3d), ref) <= TOL32
    t3i = synth.small_int(t3.shape, 103); t2i = synth.small_int(t2.shape, 104); v2i = synth.small_int(v2.shape, 105)
    t3d = dev(t3i)
    run(d, tiles, [t3d, dev(t2i), dev(v2i)])
    assert np.array_equal(host(t3d), O.ccsd_t_d1(t3i, t2i, v2i))


def test_ccsd_coverage(cuda_device):
    dims = (3, 4, 5, 3, 4, 9, 5)
    d = E.desc_builtin("ccsd_t_d1", dims)
    counts = torch.zeros(int(np.prod(dims)), dtype=torch.int32, device="cuda")
    E.coverage(d, 0, (2, 2, 2, 2, 2, 8, 2), counts)
    c = counts.cpu().numpy()
    assert c.min() == 1 and c.max() == 1


def test_ccsd_full_size_dims48_sampled(cuda_device):
    """dims 48 (config 5) with the EATSS tile: t3 = 0 start, 48.9 GB output, sampled exact dots."""
    n = 48
    d = E.desc_builtin("ccsd_t_d1", (n,))
    tiles, _ = E.select_tiles(d, E.gpu_params_query(0), 50, 4)
    t2 = synth.uniform((n, n, n, n), 110); v2 = synth.uniform((n, n, n, n), 111)
    t3d = torch.zeros(n ** 6, dtype=torch.float32, device="cuda")
    run(d, tiles, [t3d, dev(t2), dev(v2)])
    g = synth.rng(112)
    idx = np.concatenate([g.integers(0, n ** 6, 100000), np.arange(n ** 4) + 7 * n ** 5 + 3 * n ** 4])  # + one (h3,h2) plane
    got = t3d[torch.from_numpy(idx).cuda()].double().cpu().numpy()
    ref = O.ccsd_t_d1_entries((n,) * 7, idx, np.zeros(len(idx)), t2, v2)
    assert O.normwise_rel_err(got, ref) <= TOL32
    del t3d
    torch.cuda.empty_cache()


# ------------------------------------------------------------------ sweep / energy
def test_sweep_reports_energy(cuda_device):
    n = 1024
    d = E.desc_builtin("gemm", (n, n, n))
    bufs = [dev(synth.uniform((n, n), s)) for s in (1, 2, 3)]
    res = E.sweep(d, [(16, 1024, 16), (32, 32, 32)], bufs, device=0, warmup=2, min_window_s=0.2)
    for r in res:
        assert r.ms_per_run > 0 and r.tflops > 0 and r.runs >= 1
        if r.status == 0:
            assert r.joules_per_run > 0 and r.avg_watts > 50 and r.gflops_per_watt > 0


# ------------------------------------------------------------------ untiled baseline (BASELINE config 4)
@pytest.mark.parametrize("kind,n,T", [("jacobi-2d", 130, 21), ("jacobi-2d", 67, 6), ("heat-3d", 40, 6),
                                      ("heat-3d", 23, 3)])
def test_stencil_untiled_engine(cuda_device, kind, n, T):
    """The untiled engine (one thread per interior point, tile vector ignored) against the oracle, and
    the linear-field fixed point exactly; a tiled and an untiled run of one descriptor use separate
    cached graphs."""
    shape = (n, n) if kind == "jacobi-2d" else (n, n, n)
    A = synth.uniform(shape, 97); B = synth.uniform(shape, 98)
    Ar, Br = (O.jacobi2d if kind == "jacobi-2d" else O.heat3d)(A, B, T)
    d = E.desc_builtin(kind, (n,), tsteps=T)
    tiles = (16, 1024) if kind == "jacobi-2d" else (16, 16, 32)
    for engine in (1, 3, 1, 3):  # alternate: graphs cached per engine
        d.set_exec(split_pct=50, engine=engine)
        Ad, Bd = dev(A), dev(B)
        run(d, tiles, [Ad, Bd])
        assert O.normwise_rel_err(host(Ad), Ar) <= TOL32 and O.normwise_rel_err(host(Bd), Br) <= TOL32
    L = synth.linear_field(shape, (2, -3) if kind == "jacobi-2d" else (2, -3, 1), 5)
    d.set_exec(split_pct=50, engine=3)
    Ld = dev(L)
    run(d, tiles, [Ld, dev(L.copy())])
    assert np.array_equal(host(Ld), L)
    g = E.desc_builtin("gemm", (64, 64, 64))
    g.set_exec(split_pct=50, engine=3)
    with pytest.raises(E.EatssError):
        run(g, (16, 16, 16), [dev(np.zeros((64, 64))), dev(np.zeros((64, 64))), dev(np.zeros((64, 64)))])

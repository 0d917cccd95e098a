"""The 3xFP16 tcgen05 engine (engine = TENSOR_F16, tc_mma.cu): every row of A / column of B is scaled by a
power of two into fp16's range, split into hi + lo fp16 halves, accumulated as hi*hi + hi*lo + lo*hi in fp32,
and unscaled exactly in the epilogue.  Bars as for every fp32 path: small integers bit-exact for every tile,
U[-1,1) within normwise 1e-5 of the fp64 oracle -- also when rows / columns span 2^+-30 (the scaling) and
when magnitudes exceed fp16's range."""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu
E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")
F16 = 4


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(device="cuda", dtype=torch.float32)


def host(t):
    torch.cuda.synchronize()
    return t.double().cpu().numpy()


def _space():
    return [(ti, tj, tk) for ti in (128, 256) for tj in range(16, 257, 16) for tk in (16, 32, 64, 128)]


def test_f16_whole_tile_space_exact(cuda_device):
    ni, nj, nk = 300, 1100, 204
    A = synth.small_int((ni, nk), 10); B = synth.small_int((nk, nj), 11); C = synth.small_int((ni, nj), 12)
    ref = O.gemm(1.0, 1.0, C, A, B)
    As = synth.small_int((ni, nk), 13); Cs = synth.small_int((ni, ni), 14)
    refs = O.syrk(1.0, 1.0, Cs, As)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 1.0); d.set_exec(50, F16)
    ds = E.desc_builtin("syrk", (ni, nk)); ds.set_scalars(1.0, 1.0); ds.set_exec(50, F16)
    Ad, Bd, Asd = dev(A), dev(B), dev(As)
    ran = 0
    for t in _space():
        for dd, mk, r in ((d, lambda: [dev(C), Ad, Bd], ref), (ds, lambda: [dev(Cs), Asd], refs)):
            b = mk()
            try:
                E.run(dd, t, b)
            except E.EatssError as err:
                assert err.status == -5 and t[2] == 128, t  # only shared memory rejects a tile
                continue
            assert np.array_equal(host(b[0]), r), t
            ran += 1
    assert ran >= 200


@pytest.mark.parametrize("tiles", [(256, 256, 64), (128, 256, 64), (256, 96, 32), (128, 48, 128), (128, 16, 16)])
def test_f16_random_tolerance(cuda_device, tiles):
    ni, nj, nk = 260, 516, 1000
    A = synth.uniform((ni, nk), 20); B = synth.uniform((nk, nj), 21); C = synth.uniform((ni, nj), 22)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.5, 1.2); d.set_exec(50, F16)
    Cd = dev(C)
    E.run(d, tiles, [Cd, dev(A), dev(B)])
    assert O.normwise_rel_err(host(Cd), O.gemm(1.5, 1.2, C, A, B)) <= 1e-5


def test_f16_scaling_spans_the_fp32_range(cuda_device):
    """Rows of A and columns of B scaled by 2^k, k in [-30, 30] (fp16 alone covers 2^-24..2^16), plus
    entries far above fp16's maximum: the per-row / per-column exponents keep every split in range."""
    ni, nj, nk = 300, 260, 500
    g = synth.rng(31)
    A = synth.uniform((ni, nk), 32) * (2.0 ** g.integers(-30, 31, (ni, 1)))
    B = synth.uniform((nk, nj), 33) * (2.0 ** g.integers(-30, 31, (1, nj)))
    A[7] *= 1e6  # |A| up to ~1e15 > 65504
    A = A.astype(np.float32); B = B.astype(np.float32)
    C = np.zeros((ni, nj), np.float32)
    d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 0.0); d.set_exec(50, F16)
    Cd = dev(C)
    E.run(d, (256, 256, 64), [Cd, dev(A), dev(B)])
    ref = O.gemm(1.0, 0.0, C, A, B)
    out = host(Cd)
    # every row / column block on its own scale: compare entrywise against |A||B| (the dot's magnitude)
    mag = np.abs(A.astype(np.float64)) @ np.abs(B.astype(np.float64))
    assert np.max(np.abs(out - ref) / mag) <= 1e-5


def test_f16_2mm_3mm_syrk(cuda_device):
    ni, nj, nk, nl, nm = 331, 260, 296, 300, 140
    A = synth.uniform((ni, nk), 50); B = synth.uniform((nk, nj), 51)
    C = synth.uniform((nj, nl), 52); D = synth.uniform((ni, nl), 53)
    tmp_ref, D_ref = O.two_mm(1.5, 1.2, A, B, C, D)
    d = E.desc_builtin("2mm", (ni, nj, nk, nl)); d.set_scalars(1.5, 1.2); d.set_exec(50, F16)
    tmp = torch.full((ni, nj), float("nan"), device="cuda"); Dd = dev(D)
    E.run(d, (256, 256, 64), [tmp, dev(A), dev(B), dev(C), Dd])
    assert O.normwise_rel_err(host(tmp), tmp_ref) <= 1e-5 and O.normwise_rel_err(host(Dd), D_ref) <= 1e-5
    C3 = synth.uniform((nj, nm), 54); D3 = synth.uniform((nm, nl), 55)
    E_ref, F_ref, G_ref = O.three_mm(A, B, C3, D3)
    d = E.desc_builtin("3mm", (ni, nj, nk, nl, nm)); d.set_exec(50, F16)
    Eb, Fb, Gb = (torch.full(s, float("nan"), device="cuda") for s in ((ni, nj), (nj, nl), (ni, nl)))
    E.run(d, (256, 256, 64), [Eb, dev(A), dev(B), Fb, dev(C3), dev(D3), Gb])
    for got, want in ((Eb, E_ref), (Fb, F_ref), (Gb, G_ref)):
        assert O.normwise_rel_err(host(got), want) <= 1e-5
    As = synth.uniform((ni, nk), 56); Cs = synth.uniform((ni, ni), 57)
    d = E.desc_builtin("syrk", (ni, nk)); d.set_scalars(1.5, 1.2); d.set_exec(50, F16)
    Cd = dev(Cs)
    E.run(d, (256, 256, 64), [Cd, dev(As)])
    assert O.normwise_rel_err(host(Cd), O.syrk(1.5, 1.2, Cs, As)) <= 1e-5


def test_f16_model_tile_and_launch_count(cuda_device):
    d = E.desc_builtin("gemm", (4000, 4000, 4000)); d.set_exec(50, F16)
    tiles, _ = E.select_tiles(d, E.gpu_params_query(0), 50, 16, mode=3)
    assert tiles == (256, 256, 64)
    assert E.launches_per_run(d, tiles) == 3  # row / column maxima, the split / tail pre-pass, the GEMM
    ds = E.desc_builtin("syrk", (4000, 4000)); ds.set_exec(50, F16)
    assert E.launches_per_run(ds, tiles) == 3
    dc = E.desc_builtin("ccsd_t_d1", (8,)); dc.set_exec(50, F16)
    with pytest.raises(E.EatssError) as ei:
        E.run(dc, (1, 1, 1, 8, 8, 8, 8), [torch.zeros(dc.buffer_elems(i), device="cuda") for i in range(3)])
    assert ei.value.status == -5

"""The warp-alignment knob in the SIMT executor (exec.warp_align = WAF, the "SIMT length as a fraction
of the warp size") and the honest carve-out (exec.carveout_exact).

WAF permutes which (row, column) slots the lanes of a warp own, so every run must stay bit-exact on
small-integer inputs and cover every iteration point exactly once (indexing oracle)."""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu
E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")

WAFS = [4, 8, 16, 32]
TILES = [(16, 1024, 16), (32, 512, 48), (7, 13, 5), (64, 64, 64), (1024, 1024, 16), (4, 4, 4)]


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(device="cuda", dtype=torch.float32)


def host(t):
    torch.cuda.synchronize()
    return t.double().cpu().numpy()


@pytest.mark.parametrize("waf", WAFS)
@pytest.mark.parametrize("tiles", TILES)
def test_gemm_waf_small_int_exact(cuda_device, waf, tiles):
    for ni, nj, nk in ((301, 267, 259), (260, 1032, 132)):  # scalar path (ragged) / 16-byte path
        A = synth.small_int((ni, nk), 10); B = synth.small_int((nk, nj), 11); C = synth.small_int((ni, nj), 12)
        ref = O.gemm(1.0, 1.0, C, A, B)
        d = E.desc_builtin("gemm", (ni, nj, nk)); d.set_scalars(1.0, 1.0)
        d.set_exec(split_pct=50, engine=1, warp_align=waf)
        (p,) = E.plan(d, tiles)
        assert p.simt_x == waf
        Cd = dev(C)
        E.run(d, tiles, [Cd, dev(A), dev(B)])
        assert np.array_equal(host(Cd), ref), (ni, nj, nk)


@pytest.mark.parametrize("waf", WAFS)
def test_syrk_waf_small_int_exact(cuda_device, waf):
    ni, nj = 203, 157
    A = synth.small_int((ni, nj), 72); C = synth.small_int((ni, ni), 73)
    ref = O.syrk(1.0, 1.0, C, A)
    d = E.desc_builtin("syrk", (ni, nj)); d.set_scalars(1.0, 1.0)
    d.set_exec(split_pct=50, engine=1, warp_align=waf)
    Cd = dev(C)
    E.run(d, (16, 128, 16), [Cd, dev(A)])
    assert np.array_equal(host(Cd), ref)


@pytest.mark.parametrize("waf", WAFS)
@pytest.mark.parametrize("tiles,shape", [((16, 1024, 16), (70, 1100, 33)), ((32, 32, 32), (65, 33, 31)),
                                         ((5, 7, 3), (23, 19, 11)), ((1024, 1024, 4), (40, 1030, 9))])
def test_coverage_waf(cuda_device, waf, tiles, shape):
    ni, nj, nk = shape
    d = E.desc_builtin("gemm", shape)
    d.set_exec(split_pct=50, engine=1, warp_align=waf)
    counts = torch.zeros(ni * nj * nk, dtype=torch.int32, device="cuda")
    E.coverage(d, 0, tiles, counts)
    c = counts.cpu().numpy()
    assert c.min() == 1 and c.max() == 1


@pytest.mark.parametrize("split", [0, 50, 100])
def test_carveout_exact_is_reported(cuda_device, split):
    n = 512
    A = synth.uniform((n, n), 1); B = synth.uniform((n, n), 2); C = synth.uniform((n, n), 3)
    d = E.desc_builtin("gemm", (n, n, n))
    d.set_exec(split_pct=split, engine=1, carveout_exact=1)
    E.run(d, (16, 512, 16), [dev(C), dev(A), dev(B)])
    assert E.last_carveout(d) == [split]
    d.set_exec(split_pct=split, engine=1, carveout_exact=0)
    E.run(d, (16, 512, 16), [dev(C), dev(A), dev(B)])
    (cv,) = E.last_carveout(d)
    assert split <= cv <= 100
    # stencils: the time loop's carve-out (captured with the graph) is reported too
    j = E.desc_builtin("jacobi-2d", (256,), tsteps=4)
    j.set_exec(split_pct=split, engine=1, carveout_exact=1)
    Aj, Bj = synth.polybench_jacobi2d(256)
    E.run(j, (16, 128), [dev(Aj), dev(Bj)])
    torch.cuda.synchronize()
    assert E.last_carveout(j) == [split, split]


@pytest.mark.parametrize("waf", WAFS)
def test_stencils_waf_bit_identical_to_default_layout(cuda_device, waf):
    """The warp layout only changes which lane computes which point: every value is bit-identical to the
    default layout, and within tolerance of the fp64 oracle (heat-3d, jacobi-2d staged paths)."""
    n, T = 132, 6
    Aj, Bj = synth.polybench_jacobi2d(n)
    ref_A, _ = O.jacobi2d(Aj, Bj, T)
    outs = {}
    for w in (0, waf):
        d = E.desc_builtin("jacobi-2d", (n,), tsteps=T)
        d.set_exec(split_pct=50, engine=1, warp_align=w)
        Ad, Bd = dev(Aj), dev(Bj)
        E.run(d, (16, 64), [Ad, Bd])
        outs[w] = host(Ad)
    assert np.array_equal(outs[0], outs[waf])
    assert O.normwise_rel_err(outs[waf], ref_A) <= 1e-5
    m = 68
    Ah = synth.uniform((m, m, m), 7); Bh = Ah.copy()
    ref_h, _ = O.heat3d(Ah, Bh, 3)
    hs = {}
    for w in (0, waf):
        d = E.desc_builtin("heat-3d", (m,), tsteps=3)
        d.set_exec(split_pct=50, engine=1, warp_align=w)
        (p,) = E.plan(d, (16, 16, 32))[:1]
        assert p.simt_x == (w or 8)
        Ad, Bd = dev(Ah), dev(Bh)
        E.run(d, (16, 16, 32), [Ad, Bd])
        hs[w] = host(Ad)
    assert np.array_equal(hs[0], hs[waf])
    assert O.normwise_rel_err(hs[waf], ref_h) <= 1e-5

"""GPU parity of the low-dimensional PolyBench kernels (mvt, atax, bicg, gemver)
against the fp64 oracle.  Small-integer inputs keep every fp32 partial sum exact (|sum| < 2^24),
so those runs must equal the oracle bit for bit whatever the tile and the atomic summation order;
random U[-1,1) inputs are held to the fp32 normwise bar 1e-5.  The kernels are O(n^2), so the
BASELINE-size runs (n = 4000) are compared element by element in full.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu

E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")

TILES = [(16, 1024), (7, 13), (64, 96), (1, 2048), (300, 4)]


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.double().cpu().numpy()


def gen(kind, shape, seed):
    return synth.small_int(shape, seed) if kind == "int" else synth.uniform(shape, seed)


def check(kind, got, ref):
    if kind == "int":
        assert np.array_equal(got, ref)
    else:
        assert O.normwise_rel_err(got, ref) <= 1e-5


@pytest.mark.parametrize("tiles", TILES)
@pytest.mark.parametrize("kind,n", [("int", 301), ("rand", 257)])
def test_mvt(cuda_device, tiles, kind, n):
    x1, x2, y1, y2 = (gen(kind, n, 30 + k) for k in range(4))
    A = gen(kind, (n, n), 34)
    d = E.desc_builtin("mvt", (n,))
    b = [dev(x1), dev(x2), dev(y1), dev(y2), dev(A)]
    E.run(d, tiles, b)
    r1, r2 = O.mvt(x1, x2, y1, y2, A)
    check(kind, host(b[0]), r1)
    check(kind, host(b[1]), r2)


@pytest.mark.parametrize("tiles", TILES)
@pytest.mark.parametrize("kind,nx,ny", [("int", 190, 333), ("rand", 260, 124)])
def test_atax_bicg(cuda_device, tiles, kind, nx, ny):
    A = gen(kind, (nx, ny), 40)
    x = gen(kind, ny, 41)
    d = E.desc_builtin("atax", (nx, ny))
    b = [dev(np.full(ny, 7.0)), dev(np.full(nx, 7.0)), dev(A), dev(x)]  # outputs must be overwritten
    E.run(d, tiles, b)
    y, tmp = O.atax(A, x)
    check(kind, host(b[1]), tmp)
    if kind == "int":  # |y| stays < 2^24 at these sizes (oracle-certified below)
        assert np.abs(y).max() < 2 ** 24
    check(kind, host(b[0]), y)
    r, p = gen(kind, nx, 42), gen(kind, ny, 43)
    d = E.desc_builtin("bicg", (nx, ny))
    b = [dev(np.full(ny, -3.0)), dev(np.full(nx, -3.0)), dev(A), dev(r), dev(p)]
    E.run(d, tiles, b)
    s, q = O.bicg(A, r, p)
    check(kind, host(b[0]), s)
    check(kind, host(b[1]), q)


@pytest.mark.parametrize("tiles", TILES + [(816, 16)])
@pytest.mark.parametrize("kind,n", [("int", 40), ("rand", 180)])  # int: worst-case |w| < 2^24 needs n <= 40
def test_gemver(cuda_device, tiles, kind, n):
    A = gen(kind, (n, n), 50)
    vecs = [gen(kind, n, 51 + k) for k in range(8)]  # x w u1 v1 u2 v2 y z
    alpha, beta = (2.0, -1.0) if kind == "int" else (1.5, 1.2)
    d = E.desc_builtin("gemver", (n,)); d.set_scalars(alpha, beta)
    b = [dev(A)] + [dev(v) for v in vecs]
    E.run(d, tiles, b)
    An, xn, wn = O.gemver(alpha, beta, A, *vecs)
    if kind == "int":
        assert max(np.abs(An).max(), np.abs(xn).max(), np.abs(wn).max()) < 2 ** 24
    check(kind, host(b[0]), An)
    check(kind, host(b[1]), xn)
    check(kind, host(b[2]), wn)


def test_full_size_model_tiles(cuda_device):
    """n = 4000 with the model-selected tiles (B200 mode, sigma 50%, WAF 16), full comparison."""
    n = 4000
    gpu = E.gpu_params_query(0)
    A = synth.uniform((n, n), 60)
    v = [synth.uniform(n, 61 + k) for k in range(8)]
    d = E.desc_builtin("mvt", (n,))
    t, _ = E.select_tiles(d, gpu, 50, 16)
    b = [dev(v[0]), dev(v[1]), dev(v[2]), dev(v[3]), dev(A)]
    E.run(d, t, b)
    r1, r2 = O.mvt(v[0], v[1], v[2], v[3], A)
    assert O.normwise_rel_err(host(b[0]), r1) <= 1e-5 and O.normwise_rel_err(host(b[1]), r2) <= 1e-5
    d = E.desc_builtin("bicg", (n, n))
    t, _ = E.select_tiles(d, gpu, 50, 16)
    b = [dev(np.zeros(n)), dev(np.zeros(n)), dev(A), dev(v[2]), dev(v[3])]
    E.run(d, t, b)
    s, q = O.bicg(A, v[2], v[3])
    assert O.normwise_rel_err(host(b[0]), s) <= 1e-5 and O.normwise_rel_err(host(b[1]), q) <= 1e-5
    d = E.desc_builtin("gemver", (n,))
    t, _ = E.select_tiles(d, gpu, 50, 16)
    b = [dev(A)] + [dev(x) for x in v]
    E.run(d, t, b)
    An, xn, wn = O.gemver(1.5, 1.2, A, *v)
    for i, ref in ((0, An), (1, xn), (2, wn)):
        assert O.normwise_rel_err(host(b[i]), ref) <= 1e-5


def test_lowdim_fp64_run_is_rejected_and_coverage_unsupported(cuda_device):
    d = E.desc_builtin("mvt", (8,), "f64")
    with pytest.raises(E.EatssError) as ei:
        E.run(d, (4, 4), [torch.zeros(64, dtype=torch.float64, device="cuda")] * 5)
    assert ei.value.status == -5
    d = E.desc_builtin("atax", (8, 8))
    with pytest.raises(E.EatssError):
        E.coverage(d, 0, (4, 4), torch.zeros(64, dtype=torch.int32, device="cuda"))

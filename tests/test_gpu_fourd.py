"""GPU parity of the non-PolyBench 4-D kernels mttkrp and conv-2d (
readings R-N8, R-N9) against the fp64 oracle, through the C ABI.

* Small-integer inputs keep every fp32 partial sum exact (mttkrp: |B*C*D| <= 8 over <= 1320 terms;
  conv-2d: |sum| <= 16 f^2), so those runs equal the oracle bit for bit whatever the tile, the
  split of k across CTAs and the reassociation of the sums.
* U[-1,1) inputs are held to the fp32 normwise bar 1e-5 (north star).
* The BASELINE-size shapes (mttkrp 512 x 32 x 512 x 512, conv-2d 8192 with a 5 x 5 filter) run with
  the EATSS tile in the launch configuration bench.py times: mttkrp on 768 sampled outputs (each an
  exact 262,144-term fp64 sum), conv-2d on full-width row bands at the top, a tile seam and the bottom.
* The indexing oracle: eatss_coverage runs the executors' exact point mapping and
  every iteration point (i, j, k, l) / (i, j, p, q) must be visited exactly once.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu

E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.double().cpu().numpy()


def gen(kind, shape, seed, lo=-2, hi=2):
    return synth.small_int(shape, seed, lo, hi) if kind == "int" else synth.uniform(shape, seed)


def check(kind, got, ref):
    if kind == "int":
        assert np.array_equal(got, ref)
    else:
        assert O.normwise_rel_err(got, ref) <= 1e-5


# ------------------------------------------------------------------ mttkrp
MT_TILES = [(128, 32, 16, 16), (512, 32, 4, 4), (32, 32, 32, 32), (16, 8, 8, 8), (64, 16, 8, 20),
            (7, 12, 5, 9), (300, 4, 3, 64), (1, 128, 1, 4), (1024, 256, 1024, 1024)]


@pytest.mark.parametrize("tiles", MT_TILES)
@pytest.mark.parametrize("kind,dims", [("int", (70, 24, 33, 40)), ("rand", (96, 32, 40, 36)),
                                       ("int", (37, 21, 11, 30)), ("rand", (45, 136, 9, 44))])
def test_mttkrp(cuda_device, tiles, kind, dims):
    ni, nj, nk, nl = dims
    A0, B, C, D = gen(kind, (ni, nj), 1), gen(kind, (ni, nk, nl), 2), gen(kind, (nk, nj), 3), gen(kind, (nl, nj), 4)
    d = E.desc_builtin("mttkrp", dims)
    b = [dev(A0), dev(B), dev(C), dev(D)]
    E.run(d, tiles, b)
    ref = O.mttkrp(A0, B, C, D)
    check(kind, host(b[0]), ref)
    # deterministic: the split of k across CTAs is reduced in a fixed order
    b2 = [dev(A0)] + b[1:]
    E.run(d, tiles, b2)
    assert torch.equal(b[0], b2[0])


def test_mttkrp_full_size_eatss_tile(cuda_device):
    """BASELINE-shaped mttkrp with the B200-mode EATSS tile (the bench workload): split-k active."""
    dims = (512, 32, 512, 512)
    d = E.desc_builtin("mttkrp", dims)
    tiles, _ = E.select_tiles(d, E.gpu_params_query(0), 50, 16, 1)
    assert tuple(tiles) == (128, 32, 16, 16)
    assert E.plan(d, tiles)[0].passes > 1  # k split across CTAs
    ni, nj, nk, nl = dims
    A0, B, C, D = synth.uniform((ni, nj), 1), synth.uniform((ni, nk, nl), 2), synth.uniform((nk, nj), 3), \
        synth.uniform((nl, nj), 4)
    b = [dev(A0), dev(B), dev(C), dev(D)]
    E.run(d, tiles, b)
    got = host(b[0])
    g = np.random.default_rng(7)
    ii = np.concatenate([g.integers(0, ni, 700), [0, ni - 1, 127, 128, 255, 256]])
    jj = np.concatenate([g.integers(0, nj, 700), [0, nj - 1, 31, 0, 3, 4]])
    ref = O.mttkrp_entries(ii, jj, A0, B, C, D)
    assert np.linalg.norm(got[ii, jj] - ref) / np.linalg.norm(ref) <= 1e-5
    # small-integer pass at full size: exact (|B*C*D| <= 4, |sum| <= 4 * 262144 + 2 < 2^24)
    Ai, Bi, Ci, Di = (synth.small_int(x.shape, 10 + s, -2, 2) for s, x in enumerate((A0, B, C, D)))
    Ci = synth.small_int(C.shape, 12, -1, 1)
    b = [dev(Ai), dev(Bi), dev(Ci), dev(Di)]
    E.run(d, tiles, b)
    got = host(b[0])
    assert np.array_equal(got[ii, jj], O.mttkrp_entries(ii, jj, Ai, Bi, Ci, Di))


@pytest.mark.parametrize("tiles", [(128, 32, 16, 16), (5, 8, 3, 4), (4, 7, 2, 3), (64, 12, 9, 1)])
@pytest.mark.parametrize("dims", [(13, 12, 9, 10), (9, 7, 5, 6)])
def test_mttkrp_coverage(cuda_device, tiles, dims):
    d = E.desc_builtin("mttkrp", dims)
    counts = torch.zeros(int(np.prod(dims)), dtype=torch.int32, device="cuda")
    E.coverage(d, 0, tiles, counts)
    torch.cuda.synchronize()
    assert int(counts.min()) == 1 and int(counts.max()) == 1


def test_mttkrp_launch_count_and_plan(cuda_device):
    d = E.desc_builtin("mttkrp", (512, 32, 512, 512))
    p = E.plan(d, (128, 32, 16, 16))[0]
    assert (p.grid_x, p.grid_y) == (1, 4) and p.grid_z == p.passes
    assert E.launches_per_run(d, (128, 32, 16, 16)) == 2
    assert E.launches_per_run(d, (16, 32, 512, 512)) == 1  # 32 CTAs x 1 k-tile: no split


# ------------------------------------------------------------------ conv-2d
CV_TILES = [(16, 64, 5, 5), (8, 152, 5, 5), (4, 480, 4, 4), (16, 1024, 5, 5), (7, 12, 3, 3), (1, 4, 1, 1),
            (100, 8, 2, 2), (33, 36, 7, 7), (1024, 1024, 5, 5), (5, 9, 5, 5)]


@pytest.mark.parametrize("tiles", CV_TILES)
@pytest.mark.parametrize("kind,n,f", [("int", 132, 5), ("rand", 132, 5), ("int", 100, 3), ("rand", 68, 7),
                                      ("int", 67, 5), ("rand", 96, 4), ("int", 1100, 5)])
def test_conv2d(cuda_device, tiles, kind, n, f):
    inp = gen(kind, (n, n), 5, -4, 4)
    W = gen(kind, (f, f), 6, -4, 4)
    m = n - f + 1
    d = E.desc_builtin("conv-2d", (n, f))
    out = dev(np.full((m, m), 7.0))  # every output must be overwritten
    E.run(d, tiles, [out, dev(inp), dev(W)])
    check(kind, host(out), O.conv2d(inp, W))


def test_conv2d_full_size_eatss_tile(cuda_device):
    """BASELINE-shaped conv-2d (8192^2, 5x5) with the B200-mode EATSS tile (the bench workload);
    full-width bands of output rows at the top, across a tile seam and at the bottom."""
    n, f = 8192, 5
    d = E.desc_builtin("conv-2d", (n, f))
    tiles, _ = E.select_tiles(d, E.gpu_params_query(0), 50, 16, 1)
    assert tuple(tiles) == (16, 64, 5, 5)
    inp, W = synth.uniform((n, n), 5), synth.uniform((f, f), 6)
    m = n - f + 1
    out = torch.empty((m, m), dtype=torch.float32, device="cuda")
    E.run(d, tiles, [out, dev(inp), dev(W)])
    got = host(out)
    for r0, rows in ((0, 24), (4088, 24), (m - 21, 21)):
        ref = O.conv2d(inp[r0:r0 + rows + f - 1, :], W)
        assert O.normwise_rel_err(got[r0:r0 + rows], ref) <= 1e-5
    # small integers: exact over the same bands
    inp_i, W_i = synth.small_int((n, n), 7), synth.small_int((f, f), 8)
    E.run(d, tiles, [out, dev(inp_i), dev(W_i)])
    got = host(out)
    for r0, rows in ((0, 24), (m - 21, 21)):
        assert np.array_equal(got[r0:r0 + rows], O.conv2d(inp_i[r0:r0 + rows + f - 1, :], W_i))


@pytest.mark.parametrize("tiles", [(16, 64, 5, 5), (3, 8, 2, 2), (5, 9, 1, 1), (40, 4, 3, 3)])
@pytest.mark.parametrize("n,f", [(36, 5), (29, 3)])
def test_conv2d_coverage(cuda_device, tiles, n, f):
    d = E.desc_builtin("conv-2d", (n, f))
    m = n - f + 1
    counts = torch.zeros(m * m * f * f, dtype=torch.int32, device="cuda")
    E.coverage(d, 0, tiles, counts)
    torch.cuda.synchronize()
    assert int(counts.min()) == 1 and int(counts.max()) == 1


# ------------------------------------------------------------------ mttkrp on the tensor pipe
@pytest.mark.parametrize("kind,dims", [("int", (3, 32, 256, 64)), ("rand", (5, 32, 128, 96)),
                                       ("int", (2, 64, 384, 32)), ("rand", (3, 128, 128, 64))])
def test_mttkrp_tensor(cuda_device, kind, dims):
    """tcgen05 3xTF32 path at its MMA-legal tile (1, nj, 128, 32): small integers exact (|B| <= 2
    stays exact in tf32 hi; lo = 0), random data within the fp32 normwise bar."""
    ni, nj, nk, nl = dims
    A0, B, C, D = gen(kind, (ni, nj), 1), gen(kind, (ni, nk, nl), 2), gen(kind, (nk, nj), 3), gen(kind, (nl, nj), 4)
    d = E.desc_builtin("mttkrp", dims)
    d.set_exec(split_pct=50, engine=2)
    tiles = (1, nj, 128, 32)
    assert E.launches_per_run(d, tiles) == 3
    b = [dev(A0), dev(B), dev(C), dev(D)]
    E.run(d, tiles, b)
    check(kind, host(b[0]), O.mttkrp(A0, B, C, D))
    b2 = [dev(A0)] + b[1:]
    E.run(d, tiles, b2)
    assert torch.equal(b[0], b2[0])  # deterministic block-order reduction
    with pytest.raises(E.EatssError):
        E.run(d, (128, 32, 16, 16), b)  # not an MMA-legal tile: refused, no silent fallback


def test_mttkrp_tensor_full_size(cuda_device):
    dims = (512, 32, 512, 512)
    ni, nj, nk, nl = dims
    d = E.desc_builtin("mttkrp", dims)
    d.set_exec(split_pct=50, engine=2)
    A0, B, C, D = synth.uniform((ni, nj), 1), synth.uniform((ni, nk, nl), 2), synth.uniform((nk, nj), 3), \
        synth.uniform((nl, nj), 4)
    b = [dev(A0), dev(B), dev(C), dev(D)]
    E.run(d, (1, nj, 128, 32), b)
    got = host(b[0])
    g = np.random.default_rng(8)
    ii, jj = g.integers(0, ni, 600), g.integers(0, nj, 600)
    ref = O.mttkrp_entries(ii, jj, A0, B, C, D)
    assert np.linalg.norm(got[ii, jj] - ref) / np.linalg.norm(ref) <= 1e-5


# ------------------------------------------------------------------ degenerate cases
@pytest.mark.parametrize("n,f,tiles", [(16, 1, (4, 8, 1, 1)), (12, 12, (16, 64, 5, 5)), (13, 12, (1, 4, 1, 1)),
                                       (64, 5, (1024, 1024, 5, 5)), (8, 7, (16, 64, 7, 7)), (264, 5, (16, 64, 5, 5))])
def test_conv2d_degenerate(cuda_device, n, f, tiles):
    """1x1 filter (a scaled copy), filter = image (one output), two outputs per row, tiles larger than
    the output, the TMA-window path with ragged last tiles (m = 260 = 4 * 64 + 4 columns, 16 * 16 + 4 rows)."""
    inp, W = synth.small_int((n, n), 21), synth.small_int((f, f), 22)
    m = n - f + 1
    d = E.desc_builtin("conv-2d", (n, f))
    out = dev(np.full((m, m), 7.0))
    E.run(d, tiles, [out, dev(inp), dev(W)])
    assert np.array_equal(host(out), O.conv2d(inp, W))


@pytest.mark.parametrize("dims,tiles", [((1, 4, 1, 4), (128, 32, 16, 16)), ((5, 4, 1, 1), (1, 1, 1, 1)),
                                        ((3, 8, 7, 4), (1024, 1024, 1024, 1024)), ((33, 4, 2, 8), (16, 4, 1, 4)),
                                        ((2, 32, 3, 36), (128, 32, 16, 16))])
def test_mttkrp_degenerate(cuda_device, dims, tiles):
    """Single row / rank 4 / single-element reductions / tiles larger than every extent."""
    ni, nj, nk, nl = dims
    A0, B, C, D = (synth.small_int(s, 30 + i, -2, 2) for i, s in enumerate(((ni, nj), (ni, nk, nl), (nk, nj), (nl, nj))))
    d = E.desc_builtin("mttkrp", dims)
    b = [dev(A0), dev(B), dev(C), dev(D)]
    E.run(d, tiles, b)
    assert np.array_equal(host(b[0]), O.mttkrp(A0, B, C, D))
    counts = torch.zeros(ni * nj * nk * nl, dtype=torch.int32, device="cuda")
    E.coverage(d, 0, tiles, counts)
    torch.cuda.synchronize()
    assert int(counts.min()) == 1 and int(counts.max()) == 1

"""GPU parity of eatss_run_host (host buffers in, outputs copied back) against the fp64 oracle.

The row-block pipeline of gemm (B first, then A/C row blocks of whole i-tiles copied in,
computed and copied out on separate streams) must give the single-launch result: on
small-integer inputs every fp32 partial sum is exact, so the comparison is bit for bit.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu

E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")


def pinned(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).pin_memory()


@pytest.mark.parametrize("engine,tiles,shape,rb", [
    (2, (256, 256, 32), (1000, 520, 300), 3),   # tensor engine: CTA-pair row blocks, ragged last
    (2, (128, 208, 16), (700, 530, 300), 3),    # tensor engine: single-CTA tiles
    (2, (128, 128, 32), (700, 384, 96), 1),     # single block
    (1, (16, 1024, 16), (333, 1100, 70), 5),    # SIMT, ragged tiles
    (1, (32, 32, 32), (256, 256, 256), 8),
])
def test_run_host_gemm_small_int_exact(cuda_device, engine, tiles, shape, rb):
    M, N, K = shape
    A = synth.small_int((M, K), 11); B = synth.small_int((K, N), 12); C = synth.small_int((M, N), 13)
    d = E.desc_builtin("gemm", shape); d.set_scalars(1.0, 1.0); d.set_exec(50, engine)
    hA, hB, hC = pinned(A), pinned(B), pinned(C)
    E.run_host(d, tiles, [hC, hA, hB], rb)
    torch.cuda.synchronize()
    assert np.array_equal(hC.double().numpy(), O.gemm(1.0, 1.0, C, A, B))
    # a second call reuses the library's device copies; inputs refreshed from host
    hC.copy_(torch.from_numpy(C))
    E.run_host(d, tiles, [hC, hA, hB], rb)
    torch.cuda.synchronize()
    assert np.array_equal(hC.double().numpy(), O.gemm(1.0, 1.0, C, A, B))


def test_run_host_gemm_random_tolerance(cuda_device):
    M = N = K = 512
    A = synth.uniform((M, K), 21); B = synth.uniform((K, N), 22); C = synth.uniform((M, N), 23)
    d = E.desc_builtin("gemm", (M, N, K)); d.set_scalars(1.5, 1.2); d.set_exec(50, 2)
    hC = pinned(C)
    E.run_host(d, (128, 256, 32), [hC, pinned(A), pinned(B)], 4)
    torch.cuda.synchronize()
    assert O.normwise_rel_err(hC.double().numpy(), O.gemm(1.5, 1.2, C, A, B)) <= 1e-5


def test_run_host_other_builtins_match_run(cuda_device):
    """Non-pipelined path: the same result as eatss_run on device copies (outputs only copied back)."""
    n = 64
    Aj, Bj = synth.polybench_jacobi2d(n)
    dj = E.desc_builtin("jacobi-2d", (n,), tsteps=7)
    hA, hB = pinned(Aj), pinned(Bj)
    E.run_host(dj, (16, 1024), [hA, hB])
    torch.cuda.synchronize()
    Ar, Br = O.jacobi2d(Aj, Bj, 7)
    assert O.normwise_rel_err(hA.double().numpy(), Ar) <= 1e-5
    assert O.normwise_rel_err(hB.double().numpy(), Br) <= 1e-5
    dims = (8,) * 7
    t3 = synth.small_int((8,) * 6, 3); t2 = synth.small_int((8,) * 4, 4); v2 = synth.small_int((8,) * 4, 5)
    dc = E.desc_builtin("ccsd_t_d1", dims)
    h3 = pinned(t3)
    E.run_host(dc, (4, 4, 4, 4, 4, 8, 4), [h3, pinned(t2), pinned(v2)])
    torch.cuda.synchronize()
    assert np.array_equal(h3.double().numpy(), O.ccsd_t_d1(t3, t2, v2))


def test_run_host_rejects_device_buffers(cuda_device):
    d = E.desc_builtin("gemm", (8, 8, 8))
    with pytest.raises(TypeError):
        E.run_host(d, (8, 8, 8), [torch.zeros(64, device="cuda")] * 3)

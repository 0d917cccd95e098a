"""Full-size parity (BASELINE configs 2-3 at PolyBench EXTRALARGE, N = 4000, reading Q22) on
both engines, comparing WHOLE output matrices with the fp64 oracle (no sampling).

* U[-1,1) inputs (signed on purpose): normwise relative error <= 1e-5 (north star), and the
  largest elementwise error relative to the matrix's RMS magnitude is bounded too.
* Exact pass: small-integer / sparse-ternary inputs whose every partial sum the oracle certifies below
  2^24 (fp32) -- and, on the 3xTF32 tensor path, every MMA operand (chained products' intermediates)
  below 2^11 so that its lo half is exact -- must equal the oracle bit for bit.
The tiles are the ones the bench times: the SIMT pick (16,1024,16) and the tensor-mode pick (256,256,32).
"""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu
E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")

N = 4000
ENGINES = [(1, (16, 1024, 16)), (2, (256, 256, 32)), (4, (256, 256, 64))]
IDS = ["simt", "tensor", "tensor_f16"]


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(device="cuda", dtype=torch.float32)


def host(t):
    torch.cuda.synchronize()
    return t.double().cpu().numpy()


def max_rel_rms(x, ref):
    """max_ij |x - ref| / RMS(ref): the worst single entry, on the scale of the matrix."""
    rms = float(np.sqrt(np.mean(ref * ref)))
    return float(np.max(np.abs(x - ref)) / rms)


def check(x, ref, tol=1e-5):
    err = O.normwise_rel_err(x, ref)
    assert err <= tol, err
    assert max_rel_rms(x, ref) <= 50 * tol
    return err


@pytest.fixture(scope="module")
def mm_inputs():
    A = synth.uniform((N, N), 50); B = synth.uniform((N, N), 51)
    C = synth.uniform((N, N), 52); D = synth.uniform((N, N), 53)
    return A, B, C, D


@pytest.fixture(scope="module")
def ref_2mm(mm_inputs):
    A, B, C, D = mm_inputs
    return O.two_mm(1.5, 1.2, A, B, C, D)


@pytest.fixture(scope="module")
def ref_3mm(mm_inputs):
    A, B, C, D = mm_inputs
    return O.three_mm(A, B, C, D)


@pytest.mark.parametrize("engine,tiles", ENGINES, ids=IDS)
def test_gemm_4000_whole_matrix(cuda_device, mm_inputs, engine, tiles):
    A, B, C, _ = mm_inputs
    ref = O.gemm(1.5, 1.2, C, A, B)
    d = E.desc_builtin("gemm", (N, N, N)); d.set_scalars(1.5, 1.2); d.set_exec(50, engine)
    Cd = dev(C)
    E.run(d, tiles, [Cd, dev(A), dev(B)])
    check(host(Cd), ref)


@pytest.mark.parametrize("engine,tiles", ENGINES, ids=IDS)
def test_2mm_4000_whole_matrices(cuda_device, mm_inputs, ref_2mm, engine, tiles):
    A, B, C, D = mm_inputs
    tmp_ref, D_ref = ref_2mm
    d = E.desc_builtin("2mm", (N, N, N, N)); d.set_scalars(1.5, 1.2); d.set_exec(50, engine)
    tmp = torch.full((N, N), float("nan"), device="cuda"); Dd = dev(D)
    E.run(d, tiles, [tmp, dev(A), dev(B), dev(C), Dd])
    check(host(tmp), tmp_ref)
    check(host(Dd), D_ref)


@pytest.mark.parametrize("engine,tiles", ENGINES, ids=IDS)
def test_3mm_4000_whole_matrices(cuda_device, mm_inputs, ref_3mm, engine, tiles):
    A, B, C, D = mm_inputs
    Er, Fr, Gr = ref_3mm
    d = E.desc_builtin("3mm", (N, N, N, N, N)); d.set_exec(50, engine)
    bufs = [torch.full((N, N), float("nan"), device="cuda"), dev(A), dev(B),
            torch.full((N, N), float("nan"), device="cuda"), dev(C), dev(D),
            torch.full((N, N), float("nan"), device="cuda")]
    E.run(d, tiles, bufs)
    check(host(bufs[0]), Er)
    check(host(bufs[3]), Fr)
    check(host(bufs[6]), Gr)


@pytest.mark.parametrize("engine,tiles", ENGINES, ids=IDS)
def test_syrk_4000_whole_matrix(cuda_device, mm_inputs, engine, tiles):
    A, _, C, _ = mm_inputs
    ref = O.syrk(1.5, 1.2, C, A)
    d = E.desc_builtin("syrk", (N, N)); d.set_scalars(1.5, 1.2); d.set_exec(50, engine)
    Cd = dev(C)
    E.run(d, tiles, [Cd, dev(A)])
    check(host(Cd), ref)


@pytest.fixture(scope="module")
def ternary_inputs():
    # sparse {-1, 0, 1} at density 1/4 (synth.sparse_ternary): chained products stay small
    return tuple(synth.sparse_ternary((N, N), s) for s in (60, 61, 62, 63))


@pytest.mark.parametrize("engine,tiles", ENGINES, ids=IDS)
def test_2mm_4000_exact_certified(cuda_device, ternary_inputs, engine, tiles):
    A, B, C, D = ternary_inputs
    tmp_ref, D_ref = O.two_mm(1.0, 1.0, A, B, C, D)
    assert np.abs(tmp_ref).max() < 2 ** 11 and np.abs(D_ref).max() < 2 ** 24  # certificate (oracle only)
    d = E.desc_builtin("2mm", (N, N, N, N)); d.set_scalars(1.0, 1.0); d.set_exec(50, engine)
    tmp = torch.full((N, N), float("nan"), device="cuda"); Dd = dev(D)
    E.run(d, tiles, [tmp, dev(A), dev(B), dev(C), Dd])
    assert np.array_equal(host(tmp), tmp_ref)
    assert np.array_equal(host(Dd), D_ref)


@pytest.mark.parametrize("engine,tiles", ENGINES, ids=IDS)
def test_3mm_4000_exact_certified(cuda_device, ternary_inputs, engine, tiles):
    A, B, C, D = ternary_inputs
    Er, Fr, Gr = O.three_mm(A, B, C, D)
    assert max(np.abs(Er).max(), np.abs(Fr).max()) < 2 ** 11 and np.abs(Gr).max() < 2 ** 24  # certificate
    d = E.desc_builtin("3mm", (N, N, N, N, N)); d.set_exec(50, engine)
    bufs = [torch.full((N, N), float("nan"), device="cuda"), dev(A), dev(B),
            torch.full((N, N), float("nan"), device="cuda"), dev(C), dev(D),
            torch.full((N, N), float("nan"), device="cuda")]
    E.run(d, tiles, bufs)
    assert np.array_equal(host(bufs[0]), Er) and np.array_equal(host(bufs[3]), Fr)
    assert np.array_equal(host(bufs[6]), Gr)

"""Pins for the numeric oracle (oracle/oracle.c) against things other than itself.

Each test fixes the oracle to mathematics or to an independent library routine:
closed forms (identity, rank-1, integer matmul, fixed points, impulse responses
as walk counts), numpy/scipy reference routines on non-square shapes (a
transposed operand or swapped index fails them), and its own literal loop
order.  Nothing here calls the CUDA path.
"""
import numpy as np
import pytest
from scipy import signal

import synth
from oracle import numeric as O


# ------------------------------------------------------------------ gemm
def test_gemm_ikj_order_is_bit_identical_to_literal_ijk():
    # oracle.c runs i-k-j; the per-element op sequence is the literal i-j-k one.
    A = synth.uniform((37, 29), 1); B = synth.uniform((29, 41), 2); C = synth.uniform((37, 41), 3)
    a = O.gemm(1.5, 1.2, C, A, B, order="ikj")
    b = O.gemm(1.5, 1.2, C, A, B, order="ijk")
    assert np.array_equal(a, b)


def test_gemm_matches_numpy_on_nonsquare_random():
    A = synth.uniform((33, 20), 4); B = synth.uniform((20, 47), 5); C = synth.uniform((33, 47), 6)
    ref = 1.5 * (A.astype(np.float64) @ B.astype(np.float64)) + 1.2 * C.astype(np.float64)
    assert O.normwise_rel_err(O.gemm(1.5, 1.2, C, A, B), ref) < 1e-14


def test_gemm_small_int_equals_integer_matmul_exactly():
    A = synth.small_int((64, 50), 7); B = synth.small_int((50, 70), 8); C = synth.small_int((64, 70), 9)
    ref = C.astype(np.int64) + A.astype(np.int64) @ B.astype(np.int64)
    assert np.array_equal(O.gemm(1.0, 1.0, C, A, B), ref.astype(np.float64))


def test_gemm_identity_closed_form():
    # B = I  =>  C = beta*C0 + alpha*A  (exact with small ints and alpha, beta powers of 2)
    n = 40
    A = synth.small_int((n, n), 10); C = synth.small_int((n, n), 11)
    out = O.gemm(2.0, 0.5, C, A, np.eye(n))
    assert np.array_equal(out, 0.5 * C.astype(np.float64) + 2.0 * A.astype(np.float64))


def test_gemm_rank1_closed_form():
    # A = u v^T, B = w x^T  =>  A B = (v.w) u x^T
    g = synth.rng(12)
    u = g.integers(-3, 4, 23); v = g.integers(-3, 4, 17); w = g.integers(-3, 4, 17); x = g.integers(-3, 4, 31)
    A = np.outer(u, v); B = np.outer(w, x); C = np.zeros((23, 31))
    out = O.gemm(1.0, 0.0, C, A, B)
    assert np.array_equal(out, float(v @ w) * np.outer(u, x).astype(np.float64))


def test_gemm_entries_match_full():
    A = synth.uniform((30, 25), 13); B = synth.uniform((25, 19), 14); C = synth.uniform((30, 19), 15)
    full = O.gemm(1.5, 1.2, C, A, B)
    ii = np.array([0, 29, 7, 13]); jj = np.array([0, 18, 5, 11])
    assert np.array_equal(O.gemm_entries(ii, jj, C, A, B, 1.5, 1.2), full[ii, jj])


# ------------------------------------------------------------- 2mm 3mm syrk
def test_2mm_matches_numpy_nonsquare():
    A = synth.uniform((13, 11), 20); B = synth.uniform((11, 17), 21)
    C = synth.uniform((17, 19), 22); D = synth.uniform((13, 19), 23)
    tmp, Dout = O.two_mm(1.5, 1.2, A, B, C, D)
    t_ref = 1.5 * (A.astype(np.float64) @ B)
    assert O.normwise_rel_err(tmp, t_ref) < 1e-14
    assert O.normwise_rel_err(Dout, t_ref @ C.astype(np.float64) + 1.2 * D.astype(np.float64)) < 1e-14


def test_2mm_small_int_exact():
    A = synth.small_int((16, 12), 24, -1, 1); B = synth.small_int((12, 14), 25, -1, 1)
    C = synth.small_int((14, 10), 26, -1, 1); D = synth.small_int((16, 10), 27, -1, 1)
    tmp, Dout = O.two_mm(1.0, 1.0, A, B, C, D)
    ti = A.astype(np.int64) @ B.astype(np.int64)
    assert np.array_equal(tmp, ti.astype(np.float64))
    assert np.array_equal(Dout, (ti @ C.astype(np.int64) + D.astype(np.int64)).astype(np.float64))


def test_3mm_matches_integer_products():
    A = synth.small_int((9, 7), 30); B = synth.small_int((7, 11), 31)
    C = synth.small_int((11, 5), 32); D = synth.small_int((5, 13), 33)
    E, F, G = O.three_mm(A, B, C, D)
    Ei = A.astype(np.int64) @ B.astype(np.int64); Fi = C.astype(np.int64) @ D.astype(np.int64)
    assert np.array_equal(E, Ei) and np.array_equal(F, Fi) and np.array_equal(G, Ei @ Fi)


def test_syrk_matches_numpy_and_is_symmetric():
    A = synth.uniform((21, 34), 40)
    C0 = synth.uniform((21, 21), 41); C0 = (C0 + C0.T)  # symmetric start
    out = O.syrk(1.5, 1.2, C0, A)
    ref = 1.5 * (A.astype(np.float64) @ A.T.astype(np.float64)) + 1.2 * C0.astype(np.float64)
    assert O.normwise_rel_err(out, ref) < 1e-14
    assert np.array_equal(out, out.T)  # k-sum order is the same for (i,j) and (j,i)


# ------------------------------------------------------------------ stencils
def test_jacobi2d_linear_field_is_exact_fixed_point():
    n = 32
    A = synth.linear_field((n, n), (3, -2), 7); B = synth.linear_field((n, n), (1, 5), -4)
    Ao, Bo = O.jacobi2d(A, B, 10)
    assert np.array_equal(Ao, A.astype(np.float64))
    # B interior equals the field, B boundary is untouched
    assert np.array_equal(Bo[1:-1, 1:-1], A[1:-1, 1:-1].astype(np.float64))
    assert np.array_equal(Bo[0], B[0]) and np.array_equal(Bo[:, -1], B[:, -1])


def test_jacobi2d_impulse_equals_walk_counts():
    # X_T = 0.2^T * (#walks of length T with steps {0, +-e1, +-e2})  away from the boundary
    n, T = 41, 8
    A = synth.impulse((n, n), (20, 20)); B = np.zeros((n, n))
    Ao, _ = O.jacobi2d(A, B, T)
    k = np.array([[0, 1, 0], [1, 1, 1], [0, 1, 0]], dtype=np.int64)
    walks = np.array([[1]], dtype=np.int64)
    for _ in range(T):
        walks = signal.convolve2d(walks, k)
    ref = np.zeros((n, n)); r = T
    ref[20 - r:20 + r + 1, 20 - r:20 + r + 1] = walks * 0.2 ** T
    assert np.max(np.abs(Ao - ref)) < 1e-15


def test_heat3d_linear_field_is_exact_fixed_point():
    n = 12
    A = synth.linear_field((n, n, n), (2, -3, 1), 5)
    Ao, Bo = O.heat3d(A, A.copy(), 6)
    assert np.array_equal(Ao, A.astype(np.float64)) and np.array_equal(Bo, A.astype(np.float64))


def test_heat3d_impulse_equals_kernel_power():
    # one sweep: X' = 0.25 X + 0.125 * (sum of 6 face neighbours) = K/8 (*) X
    n, T = 19, 2  # 2T = 4 sweeps, support radius 4 stays inside
    c = n // 2
    A = synth.impulse((n, n, n), (c, c, c))
    Ao, Bo = O.heat3d(A, A.copy(), T)
    K = np.zeros((3, 3, 3), dtype=np.int64)
    K[1, 1, 1] = 2
    for ax in range(3):
        for s in (0, 2):
            idx = [1, 1, 1]; idx[ax] = s; K[tuple(idx)] = 1
    P = np.ones((1, 1, 1), dtype=np.int64)
    for _ in range(2 * T):
        P = signal.convolve(P, K, method="direct")
    r = 2 * T
    ref = np.zeros((n, n, n))
    ref[c - r:c + r + 1, c - r:c + r + 1, c - r:c + r + 1] = P / 8.0 ** (2 * T)
    assert np.max(np.abs(Ao - ref)) < 1e-15


# -------------------------------------------------------------- ccsd_t_d1
def test_ccsd_t_d1_matches_einsum():
    dims = (3, 4, 5, 2, 6, 7, 4)  # h3 h2 h1 p6 p5 p4 h7 (all distinct: catches swaps)
    H3, H2, H1, P6, P5, P4, H7 = dims
    t3 = synth.uniform((H3, H2, H1, P6, P5, P4), 50)
    t2 = synth.uniform((H7, P4, P5, H1), 51); v2 = synth.uniform((H3, H2, P6, H7), 52)
    out = O.ccsd_t_d1(t3, t2, v2)
    ref = t3.astype(np.float64) - np.einsum("gfec,abdg->abcdef", t2.astype(np.float64), v2.astype(np.float64))
    assert O.normwise_rel_err(out, ref) < 1e-14


def test_ccsd_t_d1_small_int_exact_and_entries():
    dims = (4, 3, 5, 4, 3, 6, 5)
    H3, H2, H1, P6, P5, P4, H7 = dims
    t3 = synth.small_int((H3, H2, H1, P6, P5, P4), 53)
    t2 = synth.small_int((H7, P4, P5, H1), 54); v2 = synth.small_int((H3, H2, P6, H7), 55)
    out = O.ccsd_t_d1(t3, t2, v2)
    ref = t3.astype(np.int64) - np.einsum("gfec,abdg->abcdef", t2.astype(np.int64), v2.astype(np.int64))
    assert np.array_equal(out, ref.astype(np.float64))
    idx = np.array([0, t3.size - 1, 123, 777])
    ent = O.ccsd_t_d1_entries(dims, idx, t3.ravel()[idx], t2, v2)
    assert np.array_equal(ent, out.ravel()[idx])


def test_normwise_error_definition():
    ref = np.array([3.0, 4.0]); x = np.array([3.0, 4.5])
    assert O.normwise_rel_err(x, ref) == pytest.approx(0.5 / 5.0)


# ---------------------------------------------------------------- low-dimensional kernels
# (PolyBench 3.2 mvt / atax / bicg / gemver, reading R-N7).  Pins: closed forms
# on rank-1 integer matrices (every value an exact integer in fp64), and integer-matrix identities.

def _ints(shape, seed, lo=-4, hi=5):
    return np.random.default_rng(seed).integers(lo, hi, size=shape).astype(np.float64)


def test_mvt_rank1_closed_form():
    n = 37
    u, v = _ints(n, 1), _ints(n, 2)
    A = np.outer(u, v)
    x1, x2, y1, y2 = _ints(n, 3), _ints(n, 4), _ints(n, 5), _ints(n, 6)
    r1, r2 = O.mvt(x1, x2, y1, y2, A)
    # x1 += A y1 = u (v . y1);  x2 += A^T y2 = v (u . y2)
    assert np.array_equal(r1, x1 + u * float(v @ y1))
    assert np.array_equal(r2, x2 + v * float(u @ y2))


def test_mvt_transposed_operand_is_not_swapped():
    """A non-symmetric integer matrix: x2 must use A^T (a swapped index fails here)."""
    A = np.triu(np.ones((5, 5)))
    y = np.arange(1.0, 6.0)
    r1, r2 = O.mvt(np.zeros(5), np.zeros(5), y, y, A)
    assert np.array_equal(r1, np.array([15.0, 14.0, 12.0, 9.0, 5.0]))   # row suffix sums
    assert np.array_equal(r2, np.array([1.0, 3.0, 6.0, 10.0, 15.0]))    # column prefix sums


def test_atax_rank1_closed_form_and_rectangular():
    nx, ny = 23, 31
    u, v, x = _ints(nx, 7), _ints(ny, 8), _ints(ny, 9)
    y, tmp = O.atax(np.outer(u, v), x)
    assert np.array_equal(tmp, u * float(v @ x))
    assert np.array_equal(y, v * float(u @ u) * float(v @ x))
    A = _ints((nx, ny), 10)
    y2, tmp2 = O.atax(A, x)
    assert np.array_equal(tmp2, A.astype(np.int64) @ x.astype(np.int64))
    assert np.array_equal(y2, A.T.astype(np.int64) @ (A.astype(np.int64) @ x.astype(np.int64)))


def test_bicg_integer_identities():
    nx, ny = 19, 29
    A, r, p = _ints((nx, ny), 11), _ints(nx, 12), _ints(ny, 13)
    s, q = O.bicg(A, r, p)
    Ai = A.astype(np.int64)
    assert np.array_equal(s, Ai.T @ r.astype(np.int64))
    assert np.array_equal(q, Ai @ p.astype(np.int64))


def test_gemver_closed_form_on_integers():
    n = 17
    A = _ints((n, n), 14)
    x, w, u1, v1, u2, v2, y, z = (_ints(n, 15 + k) for k in range(8))
    alpha, beta = 2.0, -1.0
    An, xn, wn = O.gemver(alpha, beta, A, x, w, u1, v1, u2, v2, y, z)
    Ap = A + np.outer(u1, v1) + np.outer(u2, v2)
    xp = x + beta * (Ap.T @ y) + z
    assert np.array_equal(An, Ap)
    assert np.array_equal(xn, xp)
    assert np.array_equal(wn, w + alpha * (Ap @ xp))   # w uses the UPDATED x (nest order)


# ------------------------------------------------------------------ mttkrp (reading R-N8)
def _khatri_rao(C, D):
    """Column-wise Kronecker product: row k*L + l, column j = C[k][j] * D[l][j] (textbook definition)."""
    K, J = C.shape
    L = D.shape[0]
    return (C[:, None, :] * D[None, :, :]).reshape(K * L, J)


def test_mttkrp_equals_unfolding_times_khatri_rao_on_integers():
    """MTTKRP's textbook closed form A + B_(1) (C ⊙ D) with the mode-1 unfolding B_(1) (I x KL):
    a swapped C/D, a transposed factor or a wrong unfolding order fails (K != L != J)."""
    I, J, K, L = 7, 5, 6, 4
    A0, B, C, D = _ints((I, J), 1), _ints((I, K, L), 2), _ints((K, J), 3), _ints((L, J), 4)
    got = O.mttkrp(A0, B, C, D)
    want = A0 + B.reshape(I, K * L) @ _khatri_rao(C, D)
    assert np.array_equal(got, want)
    swapped = A0 + B.reshape(I, K * L) @ _khatri_rao(np.zeros((K, J)) + C[:, ::-1], D)
    assert not np.array_equal(got, swapped)


def test_mttkrp_rank1_tensor_closed_form():
    """B = a ∘ b ∘ c (rank 1): A[i][j] = A0[i][j] + a_i (b . C[:, j]) (c . D[:, j]), exact on integers."""
    I, J, K, L = 9, 6, 8, 5
    a, b, c = _ints(I, 5), _ints(K, 6), _ints(L, 7)
    B = a[:, None, None] * b[None, :, None] * c[None, None, :]
    A0, C, D = _ints((I, J), 8), _ints((K, J), 9), _ints((L, J), 10)
    got = O.mttkrp(A0, B, C, D)
    assert np.array_equal(got, A0 + np.outer(a, (b @ C) * (c @ D)))


def test_mttkrp_brute_force_tiny_and_entries():
    I, J, K, L = 3, 4, 2, 3
    A0, B, C, D = (synth.uniform(s, seed) for s, seed in (((I, J), 1), ((I, K, L), 2), ((K, J), 3), ((L, J), 4)))
    want = A0.astype(np.float64).copy()
    for i in range(I):
        for j in range(J):
            for k in range(K):
                for l in range(L):
                    want[i, j] = want[i, j] + float(B[i, k, l]) * float(C[k, j]) * float(D[l, j])
    got = O.mttkrp(A0, B, C, D)
    assert np.array_equal(got, want)  # same operation order as written: bit-identical
    ii, jj = np.array([0, 2, 1]), np.array([3, 0, 1])
    assert np.array_equal(O.mttkrp_entries(ii, jj, A0, B, C, D), got[ii, jj])


# ------------------------------------------------------------------ conv-2d (reading R-N9)
def test_conv2d_matches_scipy_valid_correlation():
    """scipy.signal.correlate2d(mode='valid') is the textbook definition; a flipped filter
    (true convolution) or a transposed index fails on a non-symmetric filter."""
    inp = synth.uniform((23, 23), 3).astype(np.float64)
    W = synth.uniform((5, 5), 4).astype(np.float64)
    got = O.conv2d(inp, W)
    assert got.shape == (19, 19)
    np.testing.assert_allclose(got, signal.correlate2d(inp, W, mode="valid"), rtol=0, atol=1e-13)
    assert not np.allclose(got, signal.convolve2d(inp, W, mode="valid"))


def test_conv2d_delta_filter_is_an_exact_shift():
    inp = _ints((12, 12), 11)
    for p0, q0 in ((0, 0), (2, 1), (1, 3)):
        W = np.zeros((4, 4))
        W[p0, q0] = 1.0
        assert np.array_equal(O.conv2d(inp, W), inp[p0:p0 + 9, q0:q0 + 9])


def test_conv2d_linear_field_closed_form():
    """inp = a*i + b*j + d: out[i][j] = (a*i + b*j + d)*sum(W) + a*sum_p p*W[p,:] + b*sum_q q*W[:,q]."""
    n, f, a, b, d = 17, 3, 3.0, -2.0, 5.0
    i, j = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    inp = a * i + b * j + d
    W = _ints((f, f), 12)
    m = n - f + 1
    ii, jj = np.meshgrid(np.arange(m), np.arange(m), indexing="ij")
    p = np.arange(f)
    want = (a * ii + b * jj + d) * W.sum() + a * (p @ W.sum(axis=1)) + b * (p @ W.sum(axis=0))
    assert np.array_equal(O.conv2d(inp, W), want)


def test_conv2d_filter_equal_to_image_is_one_dot_product():
    inp, W = _ints((6, 6), 13), _ints((6, 6), 14)
    assert np.array_equal(O.conv2d(inp, W), np.array([[float((inp * W).sum())]]))


def test_conv2d_rectangular_band_equals_rows_of_the_square_result():
    inp, W = synth.uniform((30, 30), 15), synth.uniform((5, 5), 16)
    full = O.conv2d(inp, W)
    assert np.array_equal(O.conv2d(inp[7:7 + 10 + 4, :], W), full[7:17])
    np.testing.assert_allclose(O.conv2d(inp[:, 3:20], W), signal.correlate2d(inp[:, 3:20].astype(np.float64),
                               W.astype(np.float64), mode="valid"), rtol=0, atol=1e-13)

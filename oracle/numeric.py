"""ctypes wrappers over oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Every wrapper takes float arrays of any float dtype, promotes them to float64
(the oracle consumes exactly the device inputs promoted to fp64) and returns
float64 results.  Loop-nest definitions and citations live in oracle.c.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-shared", "-fPIC"]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so with gcc (no CUDA involved)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def lib() -> ctypes.CDLL:
    global _lib
    with _lock:
        if _lib is None:
            _lib = ctypes.CDLL(build())
            _declare(_lib)
    return _lib


_P = ctypes.c_void_p
_I = ctypes.c_int64
_D = ctypes.c_double


def _declare(L):
    L.oracle_gemm.argtypes = [_I, _I, _I, _D, _D, _P, _P, _P]
    L.oracle_gemm_ijk.argtypes = [_I, _I, _I, _D, _D, _P, _P, _P]
    L.oracle_gemm_entries.argtypes = [_I, _P, _P, _P, _I, _I, _D, _D, _P, _P, _P]
    L.oracle_2mm.argtypes = [_I, _I, _I, _I, _D, _D, _P, _P, _P, _P, _P]
    L.oracle_3mm.argtypes = [_I, _I, _I, _I, _I, _P, _P, _P, _P, _P, _P, _P]
    L.oracle_syrk.argtypes = [_I, _I, _D, _D, _P, _P]
    L.oracle_jacobi2d.argtypes = [_I, _I, _P, _P]
    L.oracle_heat3d.argtypes = [_I, _I, _P, _P]
    L.oracle_ccsd_t_d1.argtypes = [_P, _P, _P, _P]
    L.oracle_ccsd_t_d1_entries.argtypes = [_P, _I, _P, _P, _P, _P, _P]
    L.oracle_mvt.argtypes = [_I, _P, _P, _P, _P, _P]
    L.oracle_atax.argtypes = [_I, _I, _P, _P, _P, _P]
    L.oracle_bicg.argtypes = [_I, _I, _P, _P, _P, _P, _P]
    L.oracle_gemver.argtypes = [_I, _D, _D, _P, _P, _P, _P, _P, _P, _P, _P, _P]
    L.oracle_mttkrp.argtypes = [_I, _I, _I, _I, _P, _P, _P, _P]
    L.oracle_mttkrp_entries.argtypes = [_I, _P, _P, _P, _I, _I, _I, _P, _P, _P, _P]
    L.oracle_conv2d.argtypes = [_I, _I, _I, _P, _P, _P]
    L.oracle_num_threads.restype = ctypes.c_int
    for f in ("oracle_gemm", "oracle_gemm_ijk", "oracle_gemm_entries", "oracle_2mm",
              "oracle_3mm", "oracle_syrk", "oracle_jacobi2d", "oracle_heat3d",
              "oracle_ccsd_t_d1", "oracle_ccsd_t_d1_entries", "oracle_mvt", "oracle_atax", "oracle_bicg",
              "oracle_gemver", "oracle_mttkrp", "oracle_mttkrp_entries", "oracle_conv2d"):
        getattr(L, f).restype = None


def _f64(x) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(x), dtype=np.float64)


def _i64(x) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(x), dtype=np.int64)


def _p(a: np.ndarray):
    return a.ctypes.data_as(_P)


def num_threads() -> int:
    return int(lib().oracle_num_threads())


def gemm(alpha, beta, C, A, B, order: str = "ikj") -> np.ndarray:
    """C := alpha*A*B + beta*C (PolyBench 3.2 gemm). Returns a new fp64 array."""
    C = _f64(C).copy(); A = _f64(A); B = _f64(B)
    ni, nk = A.shape
    nk2, nj = B.shape
    assert nk == nk2 and C.shape == (ni, nj)
    fn = lib().oracle_gemm if order == "ikj" else lib().oracle_gemm_ijk
    fn(ni, nj, nk, float(alpha), float(beta), _p(C), _p(A), _p(B))
    return C


def gemm_entries(ii, jj, C0, A, B, alpha, beta) -> np.ndarray:
    """Values of selected gemm outputs (full-size sampled parity)."""
    ii = _i64(ii); jj = _i64(jj); A = _f64(A); B = _f64(B)
    C0 = np.asarray(C0)
    c0 = _f64(C0[ii, jj])
    out = np.empty(len(ii), dtype=np.float64)
    nk = A.shape[1]; nj = B.shape[1]
    lib().oracle_gemm_entries(len(ii), _p(ii), _p(jj), _p(c0), nj, nk, float(alpha), float(beta),
                              _p(A), _p(B), _p(out))
    return out


def two_mm(alpha, beta, A, B, C, D):
    """PolyBench 3.2 2mm. Returns (tmp, D_out)."""
    A = _f64(A); B = _f64(B); C = _f64(C); D = _f64(D).copy()
    ni, nk = A.shape; nj = B.shape[1]; nl = C.shape[1]
    assert B.shape == (nk, nj) and C.shape == (nj, nl) and D.shape == (ni, nl)
    tmp = np.empty((ni, nj), dtype=np.float64)
    lib().oracle_2mm(ni, nj, nk, nl, float(alpha), float(beta), _p(tmp), _p(A), _p(B), _p(C), _p(D))
    return tmp, D


def three_mm(A, B, C, D):
    """PolyBench 3.2 3mm. Returns (E, F, G)."""
    A = _f64(A); B = _f64(B); C = _f64(C); D = _f64(D)
    ni, nk = A.shape; nj = B.shape[1]; nm = C.shape[1]; nl = D.shape[1]
    assert B.shape == (nk, nj) and C.shape == (nj, nm) and D.shape == (nm, nl)
    E = np.empty((ni, nj)); F = np.empty((nj, nl)); G = np.empty((ni, nl))
    lib().oracle_3mm(ni, nj, nk, nl, nm, _p(E), _p(A), _p(B), _p(F), _p(C), _p(D), _p(G))
    return E, F, G


def syrk(alpha, beta, C, A) -> np.ndarray:
    """PolyBench 3.2 syrk (full square): C := alpha*A*A' + beta*C."""
    C = _f64(C).copy(); A = _f64(A)
    ni, nj = A.shape
    assert C.shape == (ni, ni)
    lib().oracle_syrk(ni, nj, float(alpha), float(beta), _p(C), _p(A))
    return C


def jacobi2d(A, B, tsteps: int):
    """PolyBench 3.2 jacobi-2d-imper (two nests per step). Returns (A, B)."""
    A = _f64(A).copy(); B = _f64(B).copy()
    n = A.shape[0]
    assert A.shape == (n, n) and B.shape == (n, n)
    lib().oracle_jacobi2d(n, int(tsteps), _p(A), _p(B))
    return A, B


def heat3d(A, B, tsteps: int):
    """PolyBench 4.x heat-3d. Returns (A, B)."""
    A = _f64(A).copy(); B = _f64(B).copy()
    n = A.shape[0]
    assert A.shape == (n, n, n) and B.shape == (n, n, n)
    lib().oracle_heat3d(n, int(tsteps), _p(A), _p(B))
    return A, B


def ccsd_t_d1(t3, t2, v2) -> np.ndarray:
    """t3[h3,h2,h1,p6,p5,p4] -= sum_h7 t2[h7,p4,p5,h1] * v2[h3,h2,p6,h7]."""
    t3 = _f64(t3).copy(); t2 = _f64(t2); v2 = _f64(v2)
    H3, H2, H1, P6, P5, P4 = t3.shape
    H7 = t2.shape[0]
    assert t2.shape == (H7, P4, P5, H1) and v2.shape == (H3, H2, P6, H7)
    d = _i64([H3, H2, H1, P6, P5, P4, H7])
    lib().oracle_ccsd_t_d1(_p(d), _p(t3), _p(t2), _p(v2))
    return t3


def ccsd_t_d1_entries(dims, idx, t3_0, t2, v2) -> np.ndarray:
    """Sampled flat t3 entries; t3_0 holds their initial values."""
    d = _i64(dims); idx = _i64(idx); t3_0 = _f64(t3_0); t2 = _f64(t2); v2 = _f64(v2)
    out = np.empty(len(idx), dtype=np.float64)
    lib().oracle_ccsd_t_d1_entries(_p(d), len(idx), _p(idx), _p(t3_0), _p(t2), _p(v2), _p(out))
    return out


def mvt(x1, x2, y1, y2, A):
    """PolyBench 3.2 mvt. Returns (x1, x2)."""
    x1 = _f64(x1).copy(); x2 = _f64(x2).copy(); A = _f64(A)
    n = x1.shape[0]
    assert A.shape == (n, n)
    lib().oracle_mvt(n, _p(x1), _p(x2), _p(_f64(y1)), _p(_f64(y2)), _p(A))
    return x1, x2


def atax(A, x):
    """PolyBench 3.2 atax: tmp = A x, y = A^T tmp (fused loop order). Returns (y, tmp)."""
    A = _f64(A); nx, ny = A.shape
    y = np.zeros(ny); tmp = np.zeros(nx)
    lib().oracle_atax(nx, ny, _p(y), _p(tmp), _p(A), _p(_f64(x)))
    return y, tmp


def bicg(A, r, p):
    """PolyBench 3.2 bicg: s = A^T r, q = A p. Returns (s, q)."""
    A = _f64(A); nx, ny = A.shape
    s = np.zeros(ny); q = np.zeros(nx)
    lib().oracle_bicg(nx, ny, _p(s), _p(q), _p(A), _p(_f64(r)), _p(_f64(p)))
    return s, q


def gemver(alpha, beta, A, x, w, u1, v1, u2, v2, y, z):
    """PolyBench 3.2 gemver. Returns (A, x, w)."""
    A = _f64(A).copy(); x = _f64(x).copy(); w = _f64(w).copy()
    n = x.shape[0]
    assert A.shape == (n, n)
    lib().oracle_gemver(n, float(alpha), float(beta), _p(A), _p(x), _p(w), _p(_f64(u1)), _p(_f64(v1)),
                        _p(_f64(u2)), _p(_f64(v2)), _p(_f64(y)), _p(_f64(z)))
    return A, x, w


def mttkrp(A, B, C, D):
    """A[i][j] += sum_k sum_l B[i][k][l]*C[k][j]*D[l][j] (reading R-N8). Returns the new A."""
    A = _f64(A).copy(); B = _f64(B); C = _f64(C); D = _f64(D)
    ni, nk, nl = B.shape; nj = A.shape[1]
    assert A.shape == (ni, nj) and C.shape == (nk, nj) and D.shape == (nl, nj)
    lib().oracle_mttkrp(ni, nj, nk, nl, _p(A), _p(B), _p(C), _p(D))
    return A


def mttkrp_entries(ii, jj, A0, B, C, D) -> np.ndarray:
    """Sampled mttkrp outputs at (ii[s], jj[s]) (full-size parity)."""
    ii = _i64(ii); jj = _i64(jj); B = _f64(B); C = _f64(C); D = _f64(D)
    a0 = _f64(np.asarray(A0)[ii, jj])
    ni, nk, nl = B.shape; nj = C.shape[1]
    out = np.empty(len(ii), dtype=np.float64)
    lib().oracle_mttkrp_entries(len(ii), _p(ii), _p(jj), _p(a0), nj, nk, nl, _p(B), _p(C), _p(D), _p(out))
    return out


def conv2d(inp, W) -> np.ndarray:
    """Valid 2-D cross-correlation out[i][j] = sum_p sum_q inp[i+p][j+q]*W[p][q] (reading R-N9);
    inp may be rectangular (row bands of a full-size check)."""
    inp = _f64(inp); W = _f64(W)
    nr, nc = inp.shape; f = W.shape[0]
    assert W.shape == (f, f) and f <= min(nr, nc)
    out = np.empty((nr - f + 1, nc - f + 1), dtype=np.float64)
    lib().oracle_conv2d(nr, nc, f, _p(out), _p(inp), _p(W))
    return out


def normwise_rel_err(x, ref) -> float:
    """||x - ref||_F / ||ref||_F in float64 (the north-star acceptance metric)."""
    x = np.asarray(x, dtype=np.float64); ref = np.asarray(ref, dtype=np.float64)
    den = np.linalg.norm(ref.ravel())
    num = np.linalg.norm((x - ref).ravel())
    return float(num / den) if den > 0 else float(num)

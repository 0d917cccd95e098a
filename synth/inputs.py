"""Seeded input generators (numpy PCG64), used by BOTH the oracle and the CUDA path.

Rules (input recipe):
  * Every array is drawn once on the host with ``numpy.random.Generator(PCG64(seed))``
    and cast to the device dtype.  The oracle consumes exactly those values promoted
    to float64, so input rounding never enters a parity error.
  * ``uniform``      U(seed): signed uniform on [-1, 1) -- the tolerance runs.
  * ``small_int``    I(seed): integers in [lo, hi] -- the bit-exact pins.
  * ``sparse_ternary``      : {-1, 0, 1} with a given density (3mm exact pins).
  * ``polybench_*``  P      : deterministic positive PolyBench-style inits (our
                              definition in the style of PolyBench/C; the paper
                              names the suite at PAPER.md:191 but prints no init).
  * ``linear_field``        : a*i + b*j (+ c*k) + d, integer coefficients.

Nothing here computes any part of a kernel or of the tile model.
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "rng",
    "uniform",
    "small_int",
    "sparse_ternary",
    "polybench_gemm",
    "polybench_jacobi2d",
    "polybench_heat3d",
    "linear_field",
    "impulse",
]


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def uniform(shape, seed: int, dtype=np.float32) -> np.ndarray:
    """U(seed): uniform on [-1, 1), cast to ``dtype``."""
    return rng(seed).uniform(-1.0, 1.0, size=shape).astype(dtype)


def small_int(shape, seed: int, lo: int = -4, hi: int = 4, dtype=np.float32) -> np.ndarray:
    """I(seed): integers uniform in [lo, hi], stored as ``dtype``."""
    return rng(seed).integers(lo, hi + 1, size=shape).astype(dtype)


def sparse_ternary(shape, seed: int, density: float = 0.25, dtype=np.float32) -> np.ndarray:
    """{-1, 0, +1} with P(nonzero) = density, signs equiprobable."""
    g = rng(seed)
    nz = g.random(size=shape) < density
    sign = np.where(g.random(size=shape) < 0.5, -1.0, 1.0)
    return (nz * sign).astype(dtype)


def polybench_gemm(ni: int, nj: int, nk: int, dtype=np.float32):
    """P init for gemm (our definition, PolyBench style): returns (C, A, B, alpha, beta)."""
    i = np.arange(ni, dtype=np.int64)[:, None]
    j = np.arange(nj, dtype=np.int64)[None, :]
    k_row = np.arange(nk, dtype=np.int64)[None, :]
    k_col = np.arange(nk, dtype=np.int64)[:, None]
    C = (((i * j + 1) % ni) / ni).astype(dtype)
    A = (((i * (k_row + 1)) % nk) / nk).astype(dtype)
    B = (((k_col * (j + 2)) % nj) / nj).astype(dtype)
    return C, A, B, 1.5, 1.2


def polybench_jacobi2d(n: int, dtype=np.float32):
    """P init for jacobi-2d: A = (i*(j+2)+2)/n, B = (i*(j+3)+3)/n."""
    i = np.arange(n, dtype=np.float64)[:, None]
    j = np.arange(n, dtype=np.float64)[None, :]
    A = ((i * (j + 2) + 2) / n).astype(dtype)
    B = ((i * (j + 3) + 3) / n).astype(dtype)
    return A, B


def polybench_heat3d(n: int, dtype=np.float32):
    """P init for heat-3d: A = B = (i + j + (n - k)) * 10 / n."""
    i = np.arange(n, dtype=np.float64)[:, None, None]
    j = np.arange(n, dtype=np.float64)[None, :, None]
    k = np.arange(n, dtype=np.float64)[None, None, :]
    A = ((i + j + (n - k)) * 10.0 / n).astype(dtype)
    return A, A.copy()


def linear_field(shape, coeffs, offset: int = 0, dtype=np.float32) -> np.ndarray:
    """f = sum_d coeffs[d] * idx_d + offset, with small integer coefficients."""
    grids = np.meshgrid(*[np.arange(s, dtype=np.int64) for s in shape], indexing="ij")
    f = np.full(shape, offset, dtype=np.int64)
    for c, g in zip(coeffs, grids):
        f = f + int(c) * g
    return f.astype(dtype)


def impulse(shape, at, value: float = 1.0, dtype=np.float32) -> np.ndarray:
    x = np.zeros(shape, dtype=dtype)
    x[tuple(at)] = value
    return x

"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NONE of the method's arithmetic (no Householder, no checksum,
no decoder): only a counter-based random generator and the structural masks
LAPACK's DGEHRD contract assumes for ilo/ihi.  Both sides of every parity test
draw their inputs from here; neither side's code lives here.

Generator spec:
  z   = splitmix64(seed XOR idx),  idx = i + j*n  (column-major linear index)
  U01 = (z >> 11) * 2**-53                       in [0, 1)
  N01 = sqrt(-2 ln(1 - U(2 idx))) * cos(2 pi U(2 idx + 1))   (Box-Muller)
The paper draws "random" matrices without naming the distribution
(Fig. 6, Table II); U(0,1) is the primary workload, N(0,1) the
secondary.
"""
from __future__ import annotations

import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_C0 = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser on uint64 (wrap-around arithmetic)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + _C0
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        z = z ^ (z >> np.uint64(31))
    return z


def _u01(seed: int, idx: np.ndarray) -> np.ndarray:
    z = splitmix64(np.uint64(seed & 0xFFFFFFFFFFFFFFFF) ^ idx.astype(np.uint64))
    return (z >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def default_seed(n: int) -> int:
    """Seed convention of SURVEY.md 8(d): 20160523 + n."""
    return 20160523 + int(n)


def matrix(n: int, seed: int | None = None, dist: str = "uniform",
           ilo: int = 1, ihi: int | None = None, chunk_cols: int = 2048) -> np.ndarray:
    """Return an n x n float64 matrix in Fortran (column-major) order.

    dist: "uniform" -> U(0,1); "normal" -> N(0,1).
    If (ilo, ihi) != (1, n) the matrix is made upper triangular in rows and
    columns 1:ilo-1 and ihi+1:n (1-based), the structure LAPACK DGEHRD assumes.
    """
    if seed is None:
        seed = default_seed(n)
    if ihi is None:
        ihi = n
    A = np.empty((n, n), dtype=np.float64, order="F")
    if n == 0:
        return A
    rows = np.arange(n, dtype=np.uint64)
    for j0 in range(0, n, chunk_cols):
        j1 = min(n, j0 + chunk_cols)
        cols = np.arange(j0, j1, dtype=np.uint64)
        idx = rows[:, None] + cols[None, :] * np.uint64(n)
        if dist == "uniform":
            A[:, j0:j1] = _u01(seed, idx)
        elif dist == "normal":
            u1 = _u01(seed, idx * np.uint64(2))
            u2 = _u01(seed, idx * np.uint64(2) + np.uint64(1))
            A[:, j0:j1] = np.sqrt(-2.0 * np.log1p(-u1)) * np.cos(2.0 * np.pi * u2)
        else:
            raise ValueError(f"unknown dist {dist!r}")
    if ilo != 1 or ihi != n:
        apply_ilo_ihi_structure(A, ilo, ihi)
    return A


def apply_ilo_ihi_structure(A: np.ndarray, ilo: int, ihi: int) -> None:
    """Zero A(i,j) (1-based) for i > j when j < ilo or i > ihi (in place)."""
    n = A.shape[0]
    i = np.arange(1, n + 1)[:, None]
    j = np.arange(1, n + 1)[None, :]
    mask = (i > j) & ((j < ilo) | (i > ihi))
    A[mask] = 0.0


def hessenberg_matrix(n: int, seed: int | None = None) -> np.ndarray:
    """A random matrix that is already upper Hessenberg (zero below the first subdiagonal)."""
    A = matrix(n, seed)
    A[np.tril_indices(n, -2)] = 0.0
    return A


def symmetric_matrix(n: int, seed: int | None = None) -> np.ndarray:
    """A random symmetric matrix (upper triangle mirrored)."""
    A = matrix(n, seed)
    S = np.triu(A) + np.triu(A, 1).T
    return np.asfortranarray(S)

"""fp64 acceptance checkers (TEST ONLY).  Tile-streamed over rows so that they also
run on large host-resident matrices.

The paper prints no accuracy numbers (PAPER.md has no "error"/"residual"/
"orthogonality"); the quantities below are the north star's (BASELINE.json):
backward error ||A - QR||_F/||A||_F, ||R - R_ref||_F/||R_ref||_F and the
orthogonality loss ||Q^T Q - I||_F.
"""
from __future__ import annotations

import numpy as np

_ROWS = 1 << 15


def _rows(m):
    for r0 in range(0, m, _ROWS):
        yield r0, min(m, r0 + _ROWS)


def backward_error(A: np.ndarray, Q: np.ndarray, R: np.ndarray) -> float:
    """||A - Q R||_F / ||A||_F in fp64 (A, Q any real dtype; widened per tile)."""
    R = np.asarray(R, dtype=np.float64)
    num = den = 0.0
    for r0, r1 in _rows(A.shape[0]):
        a = np.asarray(A[r0:r1], dtype=np.float64)
        d = a - np.asarray(Q[r0:r1], dtype=np.float64) @ R
        num += float(np.sum(d * d))
        den += float(np.sum(a * a))
    return float(np.sqrt(num / den))


def orthogonality(Q: np.ndarray) -> float:
    """||Q^T Q - I||_F in fp64."""
    n = Q.shape[1]
    G = np.zeros((n, n))
    for r0, r1 in _rows(Q.shape[0]):
        q = np.asarray(Q[r0:r1], dtype=np.float64)
        G += q.T @ q
    return float(np.linalg.norm(G - np.eye(n)))


def r_rel_error(R: np.ndarray, R_ref: np.ndarray) -> float:
    R = np.asarray(R, dtype=np.float64)
    R_ref = np.asarray(R_ref, dtype=np.float64)
    return float(np.linalg.norm(R - R_ref) / np.linalg.norm(R_ref))


def is_upper_triangular(R: np.ndarray, positive_diag: bool = True) -> bool:
    R = np.asarray(R)
    ok = bool(np.all(np.tril(R, -1) == 0))
    if positive_diag:
        ok = ok and bool(np.all(np.diag(R) > 0))
    return ok


def gram_cholesky_r(A: np.ndarray) -> np.ndarray:
    """Reference R for large inputs: R = chol(X^T X)^T with X = fp64(stored A).

    For full column rank the positive-diagonal QR is unique, so its R equals the
    Cholesky factor of the Gram matrix (accurate to ~kappa^2 * 2^-53).  The Gram
    is accumulated tile by tile (SYRK) in fp64 with numpy/LAPACK -- an
    independent library route, not the CGS recurrence."""
    n = A.shape[1]
    G = np.zeros((n, n))
    for r0, r1 in _rows(A.shape[0]):
        x = np.asarray(A[r0:r1], dtype=np.float64)
        G += x.T @ x
    return np.linalg.cholesky(G).T

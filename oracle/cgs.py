"""Plain, slow, obviously-correct classical Gram-Schmidt QR (fp64).  TEST ONLY.

Notation follows PAPER.md section 3.1: A = [a_1 | ... | a_n] (m x n, m >= n),
Q = [q_1 | ... | q_n], R upper triangular with r_ij = q_i^T a_j.
All functions take a float64 matrix X (the exact widening of the stored A) and
return (Q, R, first_breakdown_column or -1).
"""
from __future__ import annotations

from typing import NamedTuple

import numpy as np

U64 = 2.0 ** -53


class QRResult(NamedTuple):
    Q: np.ndarray
    R: np.ndarray
    breakdown: int           # first column j whose r_jj fell below tau_j, else -1


def _finish_column(u: np.ndarray, a_norm: float, m: int, unit_roundoff: float):
    """q_j = u_j / ||u_j|| (Eq. 1), with the rank-deficiency guard of
    DESIGN.md reading R4 (the paper assumes linearly independent columns)."""
    rjj = float(np.sqrt(u @ u))
    tau = m * unit_roundoff * a_norm
    if not np.isfinite(rjj) or rjj <= tau or rjj == 0.0:
        return np.zeros_like(u), 0.0, True
    return u / rjj, rjj, False


# ---------------------------------------------------------------------------------
# O1: column CGS -- Eq. (1), CGS evaluation order
# ---------------------------------------------------------------------------------
def cgs(X: np.ndarray) -> QRResult:
    """O1. For j = 1..n:  r_{<j,j} = Q_{<j}^T a_j  (every projection taken from the
    ORIGINAL column a_j -- "CGS executes row by row in (1)");
    u_j = a_j - Q_{<j} r_{<j,j};  r_jj = ||u_j||;  q_j = u_j / r_jj."""
    X = np.asarray(X, dtype=np.float64)
    m, n = X.shape
    Q = np.zeros((m, n), order="F")
    R = np.zeros((n, n), order="F")
    brk = -1
    for j in range(n):
        a = X[:, j]
        r = Q[:, :j].T @ a
        u = a - Q[:, :j] @ r
        R[:j, j] = r
        Q[:, j], R[j, j], bad = _finish_column(u, float(np.sqrt(a @ a)), m, U64)
        if bad and brk < 0:
            brk = j
    return QRResult(Q, R, brk)


# ---------------------------------------------------------------------------------
# O2: CGS2 -- CGS with the projection applied twice (north star's "CGS2 variant")
# ---------------------------------------------------------------------------------
def cgs2(X: np.ndarray) -> QRResult:
    """O2. r1 = Q^T a; u = a - Q r1; r2 = Q^T u; u -= Q r2; R[:j,j] = r1 + r2;
    r_jj = ||u||.  Each pass is the CGS step of PAPER.md:107-109."""
    X = np.asarray(X, dtype=np.float64)
    m, n = X.shape
    Q = np.zeros((m, n), order="F")
    R = np.zeros((n, n), order="F")
    brk = -1
    for j in range(n):
        a = X[:, j]
        r1 = Q[:, :j].T @ a
        u = a - Q[:, :j] @ r1
        r2 = Q[:, :j].T @ u
        u = u - Q[:, :j] @ r2
        R[:j, j] = r1 + r2
        Q[:, j], R[j, j], bad = _finish_column(u, float(np.sqrt(a @ a)), m, U64)
        if bad and brk < 0:
            brk = j
    return QRResult(Q, R, brk)


# ---------------------------------------------------------------------------------
# O3: recursive CGS -- Eq. (2)
# ---------------------------------------------------------------------------------
def rgs(X: np.ndarray, leaf: int = 32) -> QRResult:
    """O3. [A1|A2] = [Q1|Q2] [[R11, R12], [0, R22]]  (Eq. 2): "divide evenly its
    columns into two halves ... factorize A1 = Q1 R11, compute R12 = Q1^T A2,
    update A2 = A2 - Q1 R12, QR factorize the updated A2 = Q2 R22"
    (PAPER.md:115).  Nodes of width <= leaf use O1."""
    X = np.array(X, dtype=np.float64, order="F", copy=True)
    n = X.shape[1]
    R = np.zeros((n, n), order="F")
    brk = [-1]

    def rec(c0: int, c1: int):
        w = c1 - c0
        if w <= leaf:
            res = cgs(X[:, c0:c1])
            X[:, c0:c1] = res.Q
            R[c0:c1, c0:c1] = res.R
            if res.breakdown >= 0 and brk[0] < 0:
                brk[0] = c0 + res.breakdown
            return
        h = c0 + w // 2
        rec(c0, h)                                    # A1 = Q1 R11
        R12 = X[:, c0:h].T @ X[:, h:c1]               # R12 = Q1^T A2
        X[:, h:c1] -= X[:, c0:h] @ R12                # A2 = A2 - Q1 R12
        R[c0:h, h:c1] = R12
        rec(h, c1)                                    # A2 = Q2 R22

    rec(0, n)
    return QRResult(X, R, brk[0])


# ---------------------------------------------------------------------------------
# O4: blocked CGS -- PAPER.md:113 (Fig. 1 loop)
# ---------------------------------------------------------------------------------
def blocked_cgs(X: np.ndarray, b: int) -> QRResult:
    """O4. "factorize the first b columns (termed as panel). Then we have the
    factorized Q1 and let it time the rest of the matrix A2 to get R12. The next
    step is updating the rest of the matrix A2 ... repeat"."""
    X = np.array(X, dtype=np.float64, order="F", copy=True)
    n = X.shape[1]
    R = np.zeros((n, n), order="F")
    brk = -1
    for c0 in range(0, n, b):
        c1 = min(c0 + b, n)
        res = cgs(X[:, c0:c1])                        # panel
        X[:, c0:c1] = res.Q
        R[c0:c1, c0:c1] = res.R
        if res.breakdown >= 0 and brk < 0:
            brk = c0 + res.breakdown
        if c1 < n:
            R12 = X[:, c0:c1].T @ X[:, c1:]           # R12 = Q1^T A2
            X[:, c1:] -= X[:, c0:c1] @ R12            # A2 -= Q1 R12
            R[c0:c1, c1:] = R12
    return QRResult(X, R, brk)


# ---------------------------------------------------------------------------------
# O6: recursive CGS2 -- Eq. (2) with every CGS step applied twice (SURVEY.md 8 f3,
#     DESIGN.md reading R22)
# ---------------------------------------------------------------------------------
def rgs2(X: np.ndarray, leaf: int = 32) -> QRResult:
    """O6. The recursion of Eq. (2) with reorthogonalization ("CGS2",
    the stable relative of CGS):
      node:  R12 = Q1^T A2;  A2 -= Q1 R12;  S = Q1^T A2;  A2 -= Q1 S;  R12 += S
      leaf:  [Q', R'] = CGS(panel) (Eq. 1);  [Q, S] = CGS(Q');  R = S R'
    In exact arithmetic S = 0 at the nodes and S = I at the leaves, so O6 = O3."""
    X = np.array(X, dtype=np.float64, order="F", copy=True)
    n = X.shape[1]
    R = np.zeros((n, n), order="F")
    brk = [-1]

    def rec(c0: int, c1: int):
        w = c1 - c0
        if w <= leaf:
            first = cgs(X[:, c0:c1])                  # Q' R'
            second = cgs(first.Q)                     # Q' = Q S
            X[:, c0:c1] = second.Q
            R[c0:c1, c0:c1] = second.R @ first.R      # R = S R'
            b = first.breakdown if first.breakdown >= 0 else second.breakdown
            if b >= 0 and brk[0] < 0:
                brk[0] = c0 + b
            return
        h = c0 + w // 2
        rec(c0, h)
        R12 = X[:, c0:h].T @ X[:, h:c1]               # first projection
        X[:, h:c1] -= X[:, c0:h] @ R12
        S = X[:, c0:h].T @ X[:, h:c1]                 # reorthogonalization
        X[:, h:c1] -= X[:, c0:h] @ S
        R[c0:h, h:c1] = R12 + S
        rec(h, c1)

    rec(0, n)
    return QRResult(X, R, brk[0])


# ---------------------------------------------------------------------------------
# O5: precision-emulating recursive CGS (predicts the algorithmic error level)
# ---------------------------------------------------------------------------------
def _round_bf16(x: np.ndarray) -> np.ndarray:
    u = np.asarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    u = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16) << 16
    return u.astype(np.uint32).view(np.float32)


def _round_tf32_rn(x: np.ndarray) -> np.ndarray:
    u = np.asarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    u = ((u + 0xFFF + ((u >> 13) & 1)) >> 13) << 13
    return u.astype(np.uint32).view(np.float32)


def _trunc_tf32(x: np.ndarray) -> np.ndarray:
    u = np.asarray(x, dtype=np.float32).view(np.uint32) & np.uint32(0xFFFFE000)
    return u.view(np.float32)


def _store(x, mode):
    """Round fp32 values to the storage format of `mode` (RN-even)."""
    x = np.asarray(x, dtype=np.float32)
    if mode == "fp16":
        return x.astype(np.float16).astype(np.float32)
    if mode == "bf16":
        return _round_bf16(x)
    return x                                          # tf32 / tf32x3: fp32 storage


def _mm(A, B, mode):
    """fp32-accumulated product of tensor-core operands in `mode`."""
    A = np.asarray(A, dtype=np.float32)
    B = np.asarray(B, dtype=np.float32)
    if mode == "tf32":
        return _trunc_tf32(A) @ _trunc_tf32(B)
    if mode == "tf32x3":
        ah = _round_tf32_rn(A); al = _round_tf32_rn(A - ah)
        bh = _round_tf32_rn(B); bl = _round_tf32_rn(B - bh)
        return ah @ bh + (ah @ bl + al @ bh)
    return A @ B                                      # 16-bit operands are exact in fp32


def rgs_emulated(X: np.ndarray, mode: str, leaf: int = 32, reorth: bool = False) -> QRResult:
    """O5. O3 with the GPU's storage/operand rounding emulated (R5, R8,
    R9): Q and A2' stored in the storage format, R12 rounded to it as an MMA
    operand, fp32 accumulation, leaf CGS in fp32.  An error-level predictor,
    not a bitwise model (summation order differs from the GPU).  reorth=True
    emulates O6 (CGS2) the same way."""
    Xs = _store(np.asarray(X, dtype=np.float32), mode).copy(order="F")
    m, n = Xs.shape
    R = np.zeros((n, n), dtype=np.float64)

    def panel_cgs(P):
        # Eq. (1) in fp32 on the stored panel; the q_j are used in fp32 inside the leaf
        # and rounded to storage once, when the panel is written back (R20)
        P = P.astype(np.float32)
        Q = np.zeros_like(P)
        Rp = np.zeros((P.shape[1], P.shape[1]), dtype=np.float64)
        for j in range(P.shape[1]):
            a = P[:, j]
            r = Q[:, :j].T @ a
            u = a - Q[:, :j] @ r
            rjj = np.float32(np.sqrt(np.float32(u @ u)))
            Q[:, j] = u / rjj
            Rp[:j, j] = r
            Rp[j, j] = rjj
        return _store(Q, mode), Rp

    def leaf_cgs(c0, c1):
        Q, Rp = panel_cgs(Xs[:, c0:c1])
        if reorth:
            Q, S = panel_cgs(Q)
            Rp = (S.astype(np.float32) @ Rp.astype(np.float32)).astype(np.float64)
        R[c0:c1, c0:c1] = Rp
        Xs[:, c0:c1] = Q

    def project(c0, h, c1):
        R12 = _mm(Xs[:, c0:h].T, Xs[:, h:c1], mode)
        R12op = _store(R12, mode)
        Xs[:, h:c1] = _store(Xs[:, h:c1] - _mm(Xs[:, c0:h], R12op, mode), mode)
        return R12

    def rec(c0, c1):
        w = c1 - c0
        if w <= leaf:
            leaf_cgs(c0, c1)
            return
        h = c0 + w // 2
        rec(c0, h)
        R12 = project(c0, h, c1)
        if reorth:
            R12 = (R12 + project(c0, h, c1)).astype(np.float32)
        R[c0:h, h:c1] = R12
        rec(h, c1)

    rec(0, n)
    return QRResult(Xs.astype(np.float64), R, -1)

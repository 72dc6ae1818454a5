"""The paper's analytic models, written out independently of the C++ planner (TEST ONLY).

Counts are in matrix WORDS (elements), as the paper counts them;
multiply by the storage size s for bytes.
"""
from __future__ import annotations

import math


def flops(m: int, n: int) -> float:
    """BASELINE.json metric convention: 2 m n^2 flop per factorization."""
    return 2.0 * m * n * n


def recursion_inner_products(m: int, n: int, b: int) -> list[tuple[int, int, int]]:
    """Shapes (w1, m, w2) of the inner products R12 = Q1^T A2 of the recursion
    down to blocksize b (Eq. 2 applied until width <= b; PAPER.md:189 example:
    131072^2 with b = 8192 gives 8192x131072x8192 ... 65536x131072x65536)."""
    out = []

    def rec(w):
        if w <= b:
            return
        w1 = w // 2
        rec(w1)
        out.append((w1, m, w - w1))
        rec(w - w1)

    rec(n)
    return out


def recursion_flops(m: int, n: int, b: int) -> float:
    """Sum of GEMM flops (inner + outer, 2*m*w1*w2 each) plus leaf CGS flops
    (2*m*w^2 per leaf of width w).  Equals 2 m n^2 exactly when b divides the
    widths evenly (each level contributes 4 m w1 w2 = m w^2)."""
    total = 0.0

    def rec(w):
        nonlocal total
        if w <= b:
            total += 2.0 * m * w * w
            return
        w1 = w // 2
        w2 = w - w1
        rec(w1)
        total += 4.0 * m * w1 * w2
        rec(w2)

    rec(n)
    return total


# -- blocked strategy data movement, PAPER.md:139-145 -------------------------------
def blocked_iteration_words(m: int, n: int, b: int, i: int) -> tuple[int, int]:
    """Per-iteration (H2D, D2H) of the i-th panel, i = 1..k, as printed at PAPER.md:139:
    H2D = mb + mb + m(n-ib) + mb + b(n-ib) + m(n-ib);
    D2H = mb + b^2 + b(n-ib) + m(n-ib)."""
    rest = n - i * b
    h2d = m * b + m * b + m * rest + m * b + b * rest + m * rest
    d2h = m * b + b * b + b * rest + m * rest
    return h2d, d2h


def blocked_total_words(m: int, n: int, b: int) -> tuple[float, float]:
    """Closed forms PAPER.md:141 and PAPER.md:145 (n = k b):
    H2D = (k+2) m n + n^2/2 - n b/2;   D2H = 1/2 [ (k+1) m n + n^2 + n b ]."""
    k = n // b
    h2d = (k + 2) * m * n + n * n / 2 - n * b / 2
    d2h = 0.5 * ((k + 1) * m * n + n * n + n * b)
    return h2d, d2h


# -- recursive strategy, no reuse (reading R11 of PAPER.md:147-153) -------
def recursive_noreuse_words_count(m: int, n: int, b: int) -> tuple[int, int]:
    """Brute-force traversal with the paper's own per-operation accounting
    (PAPER.md:139 applied to Eq. 2): inner reads Q1 + A2 and writes R12; outer
    reads Q1 + R12 + A2 and writes A2'; a leaf reads its panel and writes Q + R11."""
    h2d = d2h = 0

    def rec(w):
        nonlocal h2d, d2h
        if w <= b:
            h2d += m * w
            d2h += m * w + w * w
            return
        w1 = w // 2
        w2 = w - w1
        rec(w1)
        h2d += m * w1 + m * w2                 # inner: Q1, A2 in
        d2h += w1 * w2                         # inner: R12 out
        h2d += m * w1 + w1 * w2 + m * w2       # outer: Q1, R12, A2 in
        d2h += m * w2                          # outer: A2' out
        rec(w2)

    rec(n)
    return h2d, d2h


def recursive_noreuse_words_closed(m: int, n: int, b: int) -> tuple[float, float]:
    """Closed form of the count above for n = k b, k = 2^L (R11):
    H2D = (2 L + 1) m n + n^2/2 - n b/2;  D2H = (L/2 + 1) m n + n^2/2 + n b/2."""
    L = int(round(math.log2(n // b)))
    h2d = (2 * L + 1) * m * n + n * n / 2 - n * b / 2
    d2h = (L / 2 + 1) * m * n + n * n / 2 + n * b / 2
    return h2d, d2h


def recursive_printed_words(m: int, n: int, b: int) -> tuple[float, float]:
    """The formulas as printed at PAPER.md:149 and PAPER.md:153 (garbled; kept to
    document the discrepancy, R11)."""
    L = math.log2(n // b)
    return 2 * (L + 1) * m * n + m * n / 2 - n * b / 2, 0.5 * L * m * n + n * n / 2


def inner_overlap_condition(rg: float, rm: float, word_bytes: int = 4) -> float:
    """the streamed inner product hides its copies when
    (4mk+4nk)/Rm < 2mnk/Rg, i.e. (square case m = n) m > 4 Rg / Rm (fp32 words)."""
    return word_bytes * rg / rm


def recursive_noreuse_split_words(m: int, n: int, b: int) -> dict:
    """The no-reuse recursive traffic split into matrix words (A / Q / A2') and R words,
    for an executor that keeps R12 resident between the two products (so the outer
    product does not re-read R12; the paper's model of PAPER.md:147 does)."""
    out = {"h2d_matrix": 0, "d2h_matrix": 0, "d2h_r": 0}

    def rec(w):
        if w <= b:
            out["h2d_matrix"] += m * w
            out["d2h_matrix"] += m * w
            out["d2h_r"] += w * w
            return
        w1 = w // 2
        w2 = w - w1
        rec(w1)
        out["h2d_matrix"] += 2 * m * (w1 + w2)      # inner + outer read Q1 and A2
        out["d2h_matrix"] += m * w2                 # outer writes A2'
        out["d2h_r"] += w1 * w2                     # R12 out once
        rec(w2)

    rec(n)
    return out


def blocked_noreuse_split_words(m: int, n: int, b: int) -> dict:
    """PAPER.md:139 per-iteration terms without the R12 re-read, and with the last
    panel (no trailing matrix) moving only its panel in and Q out."""
    k = n // b
    out = {"h2d_matrix": 0, "d2h_matrix": 0, "d2h_r": 0}
    for i in range(1, k + 1):
        rest = n - i * b
        if rest == 0:
            out["h2d_matrix"] += m * b
        else:
            out["h2d_matrix"] += m * b + m * b + m * rest + m * b + m * rest
        out["d2h_matrix"] += m * b + m * rest
        out["d2h_r"] += b * b + b * rest
    return out

"""Seeded synthetic input generators shared by the oracle and the CUDA path.

This module is the ONE thing `oracle/` and `paper_conf_icpp_zhangw21_b200/` both
use.  It holds no arithmetic of the method (no projection, no norm, no QR of the
matrix being factored): only random / structured matrix construction and the
storage-format conversions (RN-even rounding to fp16 / bf16 / fp32 words) that
define what the "stored matrix" A is.

The paper never describes the values of its test matrices (PAPER.md:235-372,
section 5); it only fixes tall host-resident shapes.
The recipes below are the build's choices, listed in DESIGN.md section 3:

* G1 ``gaussian``      -- i.i.d. N(0,1), Philox counter-based per 4096-row block so
                          that any row shard is reproducible on its own.
* G2 ``usv``           -- dense U diag(sigma) V^T with prescribed condition number.
* G4 ``hadamard``      -- first n columns of the Sylvester-Hadamard matrix / sqrt(m)
                          (orthonormal: the QR has R = I exactly).
  ``diag_scaled``      -- hadamard * diag(2^e_j) (R = D exactly).
  ``dyadic_mixed``     -- hadamard * R0, R0 banded upper triangular with small
                          dyadic entries (R = R0 exactly, every intermediate exact).

Matrices are returned column-major (Fortran order) with leading dimension m,
the layout `rgsqr_factor` consumes (include/rgsqr.h).  bf16 has no numpy dtype;
it is carried as ``numpy.uint16`` bit patterns.
"""
from __future__ import annotations

import numpy as np

ROW_BLOCK = 4096          # Philox stream granularity for G1 (rows)

DTYPES = ("fp16", "bf16", "fp32")


def storage_numpy_dtype(dtype: str):
    return {"fp16": np.float16, "bf16": np.uint16, "fp32": np.float32}[dtype]


def storage_bytes(dtype: str) -> int:
    return {"fp16": 2, "bf16": 2, "fp32": 4}[dtype]


# ----------------------------------------------------------------------------------
# storage conversions (define the stored matrix; IEEE round-to-nearest-even)
# ----------------------------------------------------------------------------------
def f32_to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """float32 -> bfloat16 bit pattern, round-to-nearest-even (finite inputs)."""
    f = np.asarray(x, dtype=np.float32)
    u = f.view(np.uint32).astype(np.uint64)          # same-itemsize view keeps order
    r = (u + 0x7FFF + ((u >> 16) & 1)) >> 16
    return r.astype(np.uint16)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (np.asarray(b, dtype=np.uint16).astype(np.uint32) << 16).view(np.float32)


def to_storage(x: np.ndarray, dtype: str, order: str = "F") -> np.ndarray:
    """Round a real array to the storage format (RN-even), column-major."""
    if dtype == "fp32":
        return np.asarray(x, dtype=np.float32, order=order)
    if dtype == "fp16":
        return np.asarray(x, dtype=np.float16, order=order)
    if dtype == "bf16":
        return np.asarray(f32_to_bf16_bits(np.asarray(x, dtype=np.float32, order=order)),
                          order=order)
    raise ValueError(dtype)


def to_float64(a: np.ndarray, dtype: str) -> np.ndarray:
    """Exact widening of a stored matrix to float64 (keeps memory order)."""
    if dtype == "bf16":
        return np.asarray(bf16_bits_to_f32(a), dtype=np.float64, order="K")
    return np.asarray(a, dtype=np.float64, order="F" if a.flags.f_contiguous else "C")


# ----------------------------------------------------------------------------------
# G1: Gaussian, Philox per row block
# ----------------------------------------------------------------------------------
def _block_rng(seed: int, block: int) -> np.random.Generator:
    return np.random.Generator(np.random.Philox(key=(int(seed) << 64) | int(block)))


def gaussian(m: int, n: int, seed: int = 1, dtype: str = "fp32", row0: int = 0,
             out: np.ndarray | None = None) -> np.ndarray:
    """G1: a_ij ~ N(0,1), rows [row0, row0+m) of the global matrix for `seed`.

    Row block b (ROW_BLOCK rows) draws its n*ROW_BLOCK normals column by column
    from Philox(key=(seed<<64)|b), so a shard that starts on a block boundary is
    bit-identical to the same rows of the unsharded matrix.
    """
    if row0 % ROW_BLOCK:
        raise ValueError("row0 must be a multiple of ROW_BLOCK")
    if out is None:
        out = np.empty((m, n), dtype=storage_numpy_dtype(dtype), order="F")

    def fill(r):
        b = (row0 + r) // ROW_BLOCK
        rows = min(ROW_BLOCK, m - r)
        blk = _block_rng(seed, b).standard_normal((n, ROW_BLOCK), dtype=np.float32)[:, :rows]
        out[r:r + rows, :] = f32_to_bf16_bits(blk.T) if dtype == "bf16" else blk.T

    starts = list(range(0, m, ROW_BLOCK))
    if m * n >= (1 << 26) and len(starts) > 1:
        # blocks are independent streams: fill them in parallel (numpy releases the GIL)
        from concurrent.futures import ThreadPoolExecutor
        import os
        with ThreadPoolExecutor(max_workers=min(len(starts), len(os.sched_getaffinity(0)))) as ex:
            list(ex.map(fill, starts))
    else:
        for r in starts:
            fill(r)
    return out


# ----------------------------------------------------------------------------------
# G4: exact-dyadic constructions built on the Sylvester-Hadamard matrix
# ----------------------------------------------------------------------------------
def _popcount_parity(x: np.ndarray) -> np.ndarray:
    x = x.astype(np.uint64)
    p = np.zeros_like(x)
    while np.any(x):
        p ^= x & 1
        x >>= 1
    return p


def hadamard(m: int, n: int) -> np.ndarray:
    """First n columns of H_m / sqrt(m), H[i,k] = (-1)^popcount(i & k), float64.

    m must be a power of 4 so that 1/sqrt(m) = 2^-j is a dyadic number: every
    entry is +-2^-j, exact in fp16 / bf16 / tf32 / fp32.
    """
    j = int(round(np.log(m) / np.log(4)))
    if 4 ** j != m:
        raise ValueError("m must be a power of 4")
    i = np.arange(m, dtype=np.uint64)[:, None]
    k = np.arange(n, dtype=np.uint64)[None, :]
    sign = 1.0 - 2.0 * _popcount_parity(i & k).astype(np.float64)
    return np.asfortranarray(sign * 2.0 ** (-j))


def diag_scaled(m: int, n: int, seed: int = 0) -> tuple[np.ndarray, np.ndarray]:
    """(A, d): A = hadamard(m, n) * diag(d), d_j = 2^e_j with e_j in [-3, 3]."""
    rng = np.random.Generator(np.random.Philox(key=(int(seed) << 64) | 0xD1A6))
    d = 2.0 ** rng.integers(-3, 4, size=n).astype(np.float64)
    return np.asfortranarray(hadamard(m, n) * d[None, :]), d


def dyadic_r0(n: int, seed: int = 0, band: int = 4) -> np.ndarray:
    """Banded upper-triangular R0: diag in {1,2}, off-diagonals in {-2,...,2}/1.

    Column sums of |R0| stay <= 2 + 2*band = 10, so with m <= 2^20 every partial
    sum of the factorization is an integer multiple of 1/m below 2^24/m: exact in
    fp32 (exact-dyadic triangular mixing).
    """
    rng = np.random.Generator(np.random.Philox(key=(int(seed) << 64) | 0xB0B0))
    r0 = np.zeros((n, n))
    for j in range(n):
        r0[j, j] = float(rng.integers(1, 3))
        for i in range(max(0, j - band), j):
            r0[i, j] = float(rng.integers(-2, 3))
    return r0


def dyadic_mixed(m: int, n: int, seed: int = 0) -> tuple[np.ndarray, np.ndarray]:
    """(A, R0): A = hadamard(m, n) @ R0 computed exactly (small integers * 2^-j)."""
    h = hadamard(m, n)
    r0 = dyadic_r0(n, seed)
    a = np.zeros((m, n), order="F")
    for j in range(n):
        lo = max(0, j - 4)
        a[:, j] = h[:, lo:j + 1] @ r0[lo:j + 1, j]     # <= 5 terms, exact in fp64
    return a, r0


def hadamard_cols(m: int, c0: int, c1: int) -> np.ndarray:
    """Columns [c0, c1) of hadamard(m, .) (float64, Fortran order), via popcount of i & k."""
    j = int(round(np.log(m) / np.log(4)))
    if 4 ** j != m:
        raise ValueError("m must be a power of 4")
    i = np.arange(m, dtype=np.uint64)[:, None]
    k = np.arange(c0, c1, dtype=np.uint64)[None, :]
    par = (np.bitwise_count(i & k) & 1).astype(np.float64)
    return np.asfortranarray((1.0 - 2.0 * par) * 2.0 ** (-j))


def dyadic_mixed_storage(m: int, n: int, seed: int = 0, dtype: str = "fp16",
                         chunk: int = 256) -> tuple[np.ndarray, np.ndarray]:
    """(A, R0) of dyadic_mixed, written column chunk by column chunk straight into the storage
    type (every entry is exact there), in parallel: for configs[2]-sized inputs whose fp64
    copy would not fit host memory.  Bit-identical to to_storage(dyadic_mixed(m, n, seed))."""
    r0 = dyadic_r0(n, seed)
    out = np.empty((m, n), dtype=storage_numpy_dtype(dtype), order="F")

    def fill(c0):
        c1 = min(n, c0 + chunk)
        lo0 = max(0, c0 - 4)
        h = hadamard_cols(m, lo0, c1)
        blk = np.empty((m, c1 - c0), order="F")
        for j in range(c0, c1):
            lo = max(0, j - 4)
            blk[:, j - c0] = h[:, lo - lo0:j + 1 - lo0] @ r0[lo:j + 1, j]
        out[:, c0:c1] = to_storage(blk, dtype)

    from concurrent.futures import ThreadPoolExecutor
    import os
    # (each worker holds ~ 2 m chunk fp64 temporaries: at most 8 workers)
    with ThreadPoolExecutor(max_workers=min(8, len(os.sched_getaffinity(0)))) as ex:
        list(ex.map(fill, range(0, n, chunk)))
    return out, r0


# ----------------------------------------------------------------------------------
# G2: dense U diag(sigma) V^T, prescribed condition number
# ----------------------------------------------------------------------------------
def usv(m: int, n: int, kappa: float, seed: int = 0) -> tuple[np.ndarray, np.ndarray]:
    """(A, sigma): A = U diag(sigma) V^T in float64, sigma_i = sqrt(m)*kappa^(-(i)/(n-1)).

    U (m x n) and V (n x n) are orthonormal bases of seeded Gaussian matrices
    (numpy Householder QR used only as a *generator* of random orthonormal
    columns).  The sqrt(m) scale keeps entries O(1) so fp16 sees no subnormals.
    """
    rng = np.random.Generator(np.random.Philox(key=(int(seed) << 64) | 0x05F0))
    u, _ = np.linalg.qr(rng.standard_normal((m, n)))
    v, _ = np.linalg.qr(rng.standard_normal((n, n)))
    expo = np.arange(n) / max(n - 1, 1)
    sigma = np.sqrt(m) * kappa ** (-expo)
    return np.asfortranarray((u * sigma[None, :]) @ v.T), sigma

"""Pins for the CPU oracle (oracle/cgs.py) against things OTHER than itself:
LAPACK Householder QR, Cholesky of the Gram matrix, closed forms, exact
constructions, and the CGS-vs-MGS stability signature."""
import numpy as np
import pytest

import oracle
from oracle import cgs, cgs2, rgs, rgs2, blocked_cgs, rgs_emulated
import rgsqr_inputs as gi


def _householder_ref(X):
    """numpy/LAPACK Householder QR with D = sign(diag R): the unique positive-diagonal QR."""
    Q, R = np.linalg.qr(X)
    d = np.sign(np.diag(R))
    return Q * d[None, :], R * d[:, None]


ALGOS = {
    "O1": lambda X: cgs(X),
    "O2": lambda X: cgs2(X),
    "O3": lambda X: rgs(X, leaf=4),
    "O3-leaf1": lambda X: rgs(X, leaf=1),
    "O4": lambda X: blocked_cgs(X, 3),
    "O6": lambda X: rgs2(X, leaf=4),
    "O6-leaf1": lambda X: rgs2(X, leaf=1),
}


@pytest.mark.parametrize("name", list(ALGOS))
@pytest.mark.parametrize("shape", [(12, 5), (40, 17), (257, 64)])
def test_matches_householder(name, shape):
    m, n = shape
    X = np.random.default_rng(m * 31 + n).standard_normal((m, n))
    Qh, Rh = _householder_ref(X)
    res = ALGOS[name](X)
    assert res.breakdown == -1
    np.testing.assert_allclose(res.R, Rh, rtol=0, atol=1e-12 * np.abs(Rh).max())
    np.testing.assert_allclose(res.Q, Qh, rtol=0, atol=1e-11)


@pytest.mark.parametrize("name", list(ALGOS))
def test_matches_gram_cholesky(name):
    X = np.random.default_rng(7).standard_normal((300, 24))
    Rc = oracle.gram_cholesky_r(X)          # independent LAPACK route
    res = ALGOS[name](X)
    assert oracle.r_rel_error(res.R, Rc) < 1e-13


def test_closed_form_n1_n2():
    rng = np.random.default_rng(3)
    a1, a2 = rng.standard_normal(9), rng.standard_normal(9)
    res = cgs(np.stack([a1, a2], axis=1))
    r11 = np.sqrt(a1 @ a1)
    r12 = (a1 @ a2) / r11
    r22 = np.sqrt(a2 @ a2 - r12 ** 2)
    np.testing.assert_allclose(res.R, [[r11, r12], [0, r22]], rtol=1e-13, atol=1e-14)
    np.testing.assert_allclose(res.Q[:, 0], a1 / r11, rtol=1e-13)
    np.testing.assert_allclose(res.Q[:, 1], (a2 - r12 * a1 / r11) / r22, rtol=1e-12)


@pytest.mark.parametrize("m,n", [(16, 8), (1024, 64), (4096, 40)])
def test_hadamard_gives_identity_exactly(m, n):
    H = gi.hadamard(m, n)
    for res in (cgs(H), rgs(H, leaf=8), blocked_cgs(H, 16), cgs2(H)):
        np.testing.assert_array_equal(res.R, np.eye(n))
        np.testing.assert_array_equal(res.Q, H)


def test_diag_scaling_gives_d_exactly():
    A, d = gi.diag_scaled(1024, 48, seed=5)
    for res in (cgs(A), rgs(A, leaf=8), blocked_cgs(A, 7)):
        np.testing.assert_array_equal(res.R, np.diag(d))


@pytest.mark.parametrize("m,n", [(256, 32), (4096, 96)])
def test_dyadic_mixing_gives_r0_exactly(m, n):
    A, R0 = gi.dyadic_mixed(m, n, seed=2)
    H = gi.hadamard(m, n)
    for res in (cgs(A), rgs(A, leaf=8), blocked_cgs(A, 12)):
        np.testing.assert_array_equal(res.R, R0)
        np.testing.assert_array_equal(res.Q, H)


@pytest.mark.parametrize("mode", ["fp16", "bf16"])
def test_emulated_dyadic_exact(mode):
    # exact-dyadic input is reproduced bitwise even with 16-bit storage
    A, R0 = gi.dyadic_mixed(4096, 128, seed=4)
    res = rgs_emulated(A, mode, leaf=32)
    np.testing.assert_array_equal(res.R, R0)


def test_cgs_not_mgs_signature():
    """CGS loses orthogonality like u*kappa^2, MGS like u*kappa, CGS2 stays O(u)
    (PAPER.md:109 'MGS is more stable').  A swapped evaluation order (MGS by
    mistake) would pass the well-conditioned pins but fail here."""
    A, _ = gi.usv(200, 20, kappa=1e6, seed=1)
    loss_cgs = oracle.orthogonality(cgs(A).Q)
    loss_cgs2 = oracle.orthogonality(cgs2(A).Q)
    # MGS for comparison, written inline (not part of the oracle)
    Q = A.copy()
    for j in range(20):
        Q[:, j] /= np.linalg.norm(Q[:, j])
        for k in range(j + 1, 20):
            Q[:, k] -= (Q[:, j] @ Q[:, k]) * Q[:, j]
    loss_mgs = oracle.orthogonality(Q)
    assert loss_cgs > 1e-6
    assert loss_mgs < 1e-8
    assert loss_cgs2 < 1e-13


def test_invariants_gaussian():
    X = gi.to_float64(gi.gaussian(4096, 256, seed=1, dtype="fp32"), "fp32")
    res = rgs(X, leaf=32)
    assert oracle.is_upper_triangular(res.R)
    assert oracle.backward_error(X, res.Q, res.R) < 1e-14
    assert oracle.orthogonality(res.Q) < 1e-12
    assert oracle.r_rel_error(res.R, cgs(X).R) < 1e-13


def test_zero_column_breakdown():
    X = np.random.default_rng(0).standard_normal((50, 6))
    X[:, 3] = 0.0
    for res in (cgs(X), rgs(X, leaf=2), blocked_cgs(X, 4)):
        assert res.breakdown == 3
        assert res.R[3, 3] == 0.0
        assert np.all(res.Q[:, 3] == 0.0)


def test_dependent_column_breakdown():
    X = np.random.default_rng(1).standard_normal((50, 6))
    X[:, 4] = X[:, 1] - 2.0 * X[:, 0]
    assert cgs(X).breakdown == 4


@pytest.mark.parametrize("mode,tol", [("fp16", 5e-3), ("bf16", 5e-3), ("tf32", 5e-3), ("tf32x3", 1e-5)])
def test_emulation_error_levels(mode, tol):
    """O5 converges to O3 as precision increases; its error levels bracket the
    north-star tolerances (BASELINE.json) for Gaussian input."""
    X = gi.to_float64(gi.gaussian(2048, 128, seed=1, dtype="fp32"), "fp32")
    ref = rgs(X, leaf=32)
    res = rgs_emulated(X, mode, leaf=32)
    be = oracle.backward_error(X, res.Q, res.R)
    assert be < tol
    assert oracle.r_rel_error(res.R, ref.R) < tol


def test_storage_roundtrip():
    x = np.array([1.0, 1.0 + 2 ** -8, 1.0 + 3 * 2 ** -9, -3.140625, 65504.0], dtype=np.float32)
    b = gi.to_storage(x, "bf16")
    back = gi.bf16_bits_to_f32(b)
    assert back[0] == 1.0
    assert back[1] == 1.0                      # tie -> even
    assert back[2] == 1.0 + 2 ** -7            # 1.5 ulp -> round up
    assert back[3] == -3.140625


def test_gaussian_shard_reproducible():
    full = gi.gaussian(3 * gi.ROW_BLOCK, 16, seed=9, dtype="fp16")
    part = gi.gaussian(gi.ROW_BLOCK, 16, seed=9, dtype="fp16", row0=gi.ROW_BLOCK)
    np.testing.assert_array_equal(full[gi.ROW_BLOCK:2 * gi.ROW_BLOCK], part)


def test_rgs2_orthogonality_signature():
    """O6 (recursive CGS2) keeps O(u) orthogonality where CGS (O3) loses u*kappa^2:
    the property that makes it the reorthogonalized variant.  A
    missing second projection at the nodes or a missing second leaf pass fails here."""
    A, _ = gi.usv(512, 64, kappa=1e7, seed=2)
    loss_rgs = oracle.orthogonality(rgs(A, leaf=8).Q)
    loss_rgs2 = oracle.orthogonality(rgs2(A, leaf=8).Q)
    assert loss_rgs > 1e-7            # measured 9.7e-7 (u kappa^2 = 1e-2 is the worst case)
    assert loss_rgs2 < 1e-12          # measured 3.8e-13
    # a version with only the node reorthogonalization (single-pass leaves) is not enough
    X = np.array(A, order="F", copy=True)
    res = rgs2(A, leaf=64)          # one leaf = panel twice, no nodes
    assert oracle.orthogonality(res.Q) < 1e-13
    # and R is still the unique positive-diagonal R (Gram-Cholesky of the input, kappa^2 u ~ 1e-2
    # is too large for that route, so compare with Householder)
    _, Rh = _householder_ref(X)
    assert oracle.r_rel_error(rgs2(A, leaf=8).R, Rh) < 1e-8


def test_rgs2_dyadic_exact():
    # exact-dyadic input: the second projections are exactly 0 and the second leaf passes
    # exactly I, so O6 reproduces R0 and Q = H bitwise, like O3
    A, R0 = gi.dyadic_mixed(1024, 96, seed=5)
    res = rgs2(A, leaf=16)
    np.testing.assert_array_equal(res.R, R0)
    np.testing.assert_array_equal(res.Q, gi.hadamard(1024, 96))


@pytest.mark.parametrize("mode", ["fp16", "tf32x3"])
def test_emulated_reorth_levels(mode):
    """O5 with reorth=True: at kappa = 1e3 CGS2 keeps orthogonality at the storage level
    (the GPU CGS2 test thresholds come from here), single-pass CGS does not."""
    A, _ = gi.usv(2048, 128, kappa=1e3, seed=3)
    X = gi.to_float64(gi.to_storage(A.astype(np.float32), "fp16" if mode == "fp16" else "fp32"),
                      "fp16" if mode == "fp16" else "fp32")
    one = oracle.orthogonality(rgs_emulated(X, mode, leaf=32).Q)
    two = oracle.orthogonality(rgs_emulated(X, mode, leaf=32, reorth=True).Q)
    if mode == "fp16":
        assert one > 0.1 and two < 0.05
    else:
        assert one > 1e-4 and two < 1e-5
    ref = rgs(X, leaf=32)
    assert oracle.r_rel_error(rgs_emulated(X, mode, leaf=32, reorth=True).R, ref.R) < (5e-3 if mode == "fp16" else 1e-5)

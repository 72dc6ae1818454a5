"""Degenerate and ragged shapes through the C ABI, both paths (rgsqr_factor from host buffers,
rgsqr_factor_device), against the oracle; argument validation (include/rgsqr.h preconditions:
1 <= n <= m, lda >= m, lda * sizeof(elem) % 16 == 0, non-null outputs)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from tests.gpu_util import to_dev, from_dev  # noqa: E402

STOR = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32", "tf32x3": "fp32"}
TOL = {"fp16": 5e-3, "bf16": 5e-3, "tf32": 5e-3, "tf32x3": 1e-5}


@pytest.fixture(scope="module")
def h():
    from paper_conf_icpp_zhangw21_b200 import Handle
    hd = Handle(0)
    yield hd
    hd.close()


def _lda(m, st):
    e = 2 if st != "fp32" else 4
    q = 16 // e
    return (m + q - 1) // q * q


def host_factor(h, A, prec, budget=0):
    m, n = A.shape
    st = STOR[prec]
    lda = _lda(m, st)
    Ap = np.zeros((lda, n), dtype=A.dtype, order="F")
    Ap[:m] = A
    Q = np.zeros_like(Ap, order="F")
    R = np.full((n, n), np.nan, dtype=np.float32, order="F")
    rc = h.factor(Ap, lda, m, n, Q, R, precision=prec, budget=budget)
    return rc, gi.to_float64(np.asfortranarray(Q[:m]), st), R.astype(np.float64)


def device_factor(h, A, prec):
    m, n = A.shape
    st = STOR[prec]
    lda = _lda(m, st)
    Ad = to_dev(A, st)
    if lda != m:
        Ap = torch.zeros((n, lda), dtype=Ad.dtype, device="cuda")
        Ap[:, :m] = Ad
        Ad = Ap
    R = torch.full((n, n), float("nan"), dtype=torch.float32, device="cuda")
    rc = h.factor_device(Ad, lda, m, n, Ad, R, precision=prec)
    return rc, from_dev(Ad[:, :m]), R.cpu().numpy().T.astype(np.float64)


def check(X, Q, R, prec, leaf=64):
    ref = oracle.rgs(X, leaf=leaf)
    assert oracle.is_upper_triangular(R)
    assert np.all(np.diag(R) > 0)
    assert oracle.backward_error(X, Q, R) <= TOL[prec]
    assert oracle.r_rel_error(R, ref.R) <= TOL[prec]
    return ref


@pytest.mark.parametrize("path", ["host", "device"])
@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32", "tf32x3"])
def test_single_column(h, path, prec):
    """n = 1: R = ||a||, Q = a / ||a|| (the leaf's only column; Eq. 1 with no projections)."""
    st = STOR[prec]
    A = gi.gaussian(5000, 1, seed=11, dtype=st)
    X = gi.to_float64(A, st)
    rc, Q, R = (host_factor if path == "host" else device_factor)(h, A, prec)
    assert rc == 0
    nrm = np.linalg.norm(X[:, 0])
    assert abs(R[0, 0] - nrm) <= 1e-6 * nrm
    u = {"fp16": 2 ** -11, "bf16": 2 ** -8, "fp32": 2 ** -24}[st]
    assert np.max(np.abs(Q[:, 0] - X[:, 0] / nrm)) <= 2 * u * np.max(np.abs(X[:, 0])) / nrm + 1e-7


@pytest.mark.parametrize("path", ["host", "device"])
@pytest.mark.parametrize("m,n", [(1000, 37), (777, 2), (4099, 65), (9999, 129), (12347, 1000)])
def test_ragged_shapes(h, path, m, n):
    """m not a multiple of 8 (lda padded), n prime / just past a leaf or split boundary."""
    A = gi.gaussian(m, n, seed=12, dtype="fp16")
    X = gi.to_float64(A, "fp16")
    rc, Q, R = (host_factor if path == "host" else device_factor)(h, A, "fp16")
    assert rc == 0
    check(X, Q, R, "fp16")


@pytest.mark.parametrize("prec", ["fp16", "tf32"])
def test_square(h, prec):
    """m = n (the paper's square Table 4 shapes, at a small size): kappa 3 U Sigma V^T."""
    st = STOR[prec]
    A64, _ = gi.usv(512, 512, kappa=3.0, seed=13)
    A = gi.to_storage(A64, st)
    X = gi.to_float64(A, st)
    for path in (host_factor, device_factor):
        rc, Q, R = path(h, A, prec)
        assert rc == 0
        check(X, Q, R, prec)


def test_ragged_host_out_of_core(h):
    """A ragged shape under a budget small enough to force the out-of-core node (streamed tiles with a
    partial last tile)."""
    m, n = 30011, 700
    A = gi.gaussian(m, n, seed=14, dtype="fp16")
    X = gi.to_float64(A, "fp16")
    rc, Q, R = host_factor(h, A, "fp16", budget=24 << 20)
    assert rc == 0
    assert h.stats()["n_ooc_nodes"] >= 1
    check(X, Q, R, "fp16")


def test_invalid_arguments(h):
    from paper_conf_icpp_zhangw21_b200.rgsqr import RgsqrError
    A = np.asfortranarray(gi.gaussian(64, 8, seed=15, dtype="fp16"))
    Q = np.zeros_like(A, order="F")
    R = np.zeros((8, 8), dtype=np.float32, order="F")
    bad = [
        dict(lda=64, m=64, n=0),      # n < 1
        dict(lda=64, m=4, n=8),       # m < n
        dict(lda=32, m=64, n=8),      # lda < m
        dict(lda=60, m=56, n=8),      # lda * 2 bytes not a multiple of 16
    ]
    for b in bad:
        with pytest.raises(RgsqrError) as ei:
            h.factor(A, b["lda"], b["m"], b["n"], Q, R, precision="fp16")
        assert ei.value.status == -1, b
    with pytest.raises(RgsqrError) as ei:
        h.factor(A, 64, 64, 8, Q, 0, precision="fp16")   # null R_out
    assert ei.value.status == -1
    # the handle stays usable after rejected calls
    rc, Qg, Rg = host_factor(h, A, "fp16")
    assert rc == 0
    check(gi.to_float64(A, "fp16"), Qg, Rg, "fp16")


@pytest.mark.parametrize("prec", ["fp16", "tf32"])
@pytest.mark.parametrize("tiling,block", [(0, 2048), (1, 128)])
def test_ooc_gemms_ragged_m(h, prec, tiling, block):
    """The standalone OOC GEMMs (Tables 1/2 operations) with m not a multiple of the 16-byte row quantum
    (lda padded): R12 = Q1^T A2 and A2 - Q1 R12 against fp64 products of the stored operands (bounds as
    tests/test_gpu_ooc_gemm.py)."""
    st = STOR[prec]
    m, w1, w2 = 20011, 192, 264
    lda = _lda(m, st)
    Q = np.zeros((lda, w1), dtype=gi.storage_numpy_dtype(st), order="F")
    A = np.zeros((lda, w2), dtype=gi.storage_numpy_dtype(st), order="F")
    Q[:m] = gi.gaussian(m, w1, seed=21, dtype=st)
    A[:m] = gi.gaussian(m, w2, seed=22, dtype=st)
    Xq, Xa = gi.to_float64(np.asfortranarray(Q[:m]), st), gi.to_float64(np.asfortranarray(A[:m]), st)
    c = 1e-4 if st != "fp32" else 2e-3
    budget = (48 << 20) * (2 if st == "fp32" else 1)
    R = np.full((w1, w2), np.nan, dtype=np.float32, order="F")
    h.ooc_inner(Q, lda, A, lda, m, w1, w2, R, w1, precision=prec, tiling=tiling, block=block, budget=budget)
    assert np.all(np.abs(R - Xq.T @ Xa) <= c * (np.abs(Xq).T @ np.abs(Xa)))
    Rin = np.asfortranarray((np.random.default_rng(2).standard_normal((w1, w2)) / np.sqrt(w1)).astype(np.float32))
    Rop = gi.to_float64(gi.to_storage(Rin.astype(np.float64), st), st)
    A2 = np.array(A, order="F", copy=True)
    h.ooc_outer(Q, lda, Rin, w1, A2, lda, m, w1, w2, precision=prec, tiling=tiling, block=block, budget=budget)
    got = gi.to_float64(np.asfortranarray(A2[:m]), st)
    ref = Xa - Xq @ Rop
    u = {"fp16": 2.0 ** -11, "fp32": 2.0 ** -24}[st]
    bound = u * np.abs(ref) + c * (np.abs(Xq) @ np.abs(Rop)) + 1e-30
    assert np.all(np.abs(got - ref) <= bound)
    assert np.all(A2[m:] == A[m:])   # rows past m untouched


@pytest.mark.parametrize("path", ["host", "device"])
@pytest.mark.parametrize("prec", ["tf32", "tf32x3"])
@pytest.mark.parametrize("m,n", [(777, 40), (4099, 65)])
def test_ragged_shapes_fp32_storage(h, path, prec, m, n):
    """fp32 storage with m % 4 != 0: the TF32X3 hi / lo operand copies get a padded leading dimension."""
    st = STOR[prec]
    A = gi.gaussian(m, n, seed=16, dtype=st)
    X = gi.to_float64(A, st)
    rc, Q, R = (host_factor if path == "host" else device_factor)(h, A, prec)
    assert rc == 0
    check(X, Q, R, prec)


@pytest.mark.parametrize("path", ["host", "device"])
@pytest.mark.parametrize("m,n", [(1, 1), (8, 8), (16, 3), (100, 100)])
def test_tiny(h, path, m, n):
    """Smallest problems: a 1 x 1 matrix (R = |a|, Q = sign(a)), tiny square and tiny tall ones."""
    A64, _ = gi.usv(m, n, kappa=2.0, seed=17) if n > 1 else (np.array([[-3.0]] * m), None)
    A = gi.to_storage(A64, "fp32")
    X = gi.to_float64(A, "fp32")
    rc, Q, R = (host_factor if path == "host" else device_factor)(h, A, "tf32x3")
    assert rc == 0
    check(X, Q, R, "tf32x3")


@pytest.mark.parametrize("leaf", [8, 16, 24, 32])
def test_leaf_width_option(h, leaf):
    """RGSQR_OPT_LEAF_WIDTH (reading R3): narrower leaves give the same factorization within tolerance."""
    A = gi.gaussian(8192, 200, seed=18, dtype="fp16")
    X = gi.to_float64(A, "fp16")
    h.set_option("leaf_width", leaf)
    try:
        rc, Q, R = device_factor(h, A, "fp16")
    finally:
        h.set_option("leaf_width", 64)
    assert rc == 0
    check(X, Q, R, "fp16", leaf=leaf)
    assert h.stats()["n_leaf_launches"] >= 200 // leaf


@pytest.mark.parametrize("algo,reorth,prec", [(1, 0, "fp16"), (2, 0, "fp16"), (0, 1, "fp16"), (0, 0, "tf32x3"),
                                              (1, 0, "tf32"), (2, 1, "bf16")])
def test_ragged_out_of_core_modes(h, algo, reorth, prec):
    """Ragged m and n under an out-of-core budget through the blocked (1) / fused-blocked (2) algorithms,
    CGS2 and TF32X3: every executor mode with a partial last row tile and odd widths."""
    st = STOR[prec]
    m, n = 20011, 333
    A = gi.gaussian(m, n, seed=19, dtype=st)
    X = gi.to_float64(A, st)
    h.set_option("algo", algo)
    h.set_option("block_cols", 128)
    h.set_option("reorth", reorth)
    try:
        budget = (12 << 20) * (2 if st == "fp32" else 1) * (3 if prec == "tf32x3" else 1)
        rc, Q, R = host_factor(h, A, prec, budget=budget)
        ooc = h.stats()["n_ooc_nodes"]
    finally:
        h.set_option("algo", 0)
        h.set_option("block_cols", 8192)
        h.set_option("reorth", 0)
    assert rc == 0
    assert algo != 0 or ooc >= 1
    ref = oracle.rgs(X, leaf=64)
    assert oracle.is_upper_triangular(R)
    assert oracle.backward_error(X, Q, R) <= TOL[prec]
    assert oracle.r_rel_error(R, ref.R) <= max(TOL[prec], 1e-5)


@pytest.mark.parametrize("path", ["host", "device"])
def test_dependent_column_warning(h, path):
    """Reading R4 (PAPER.md:103 assumes independent columns): a column equal to an earlier one leaves
    u_j at rounding level, r_jj <= m u ||a_j|| -> q_j = 0, r_jj = 0, RGSQR_WARN_RANK_DEFICIENT (1) and the
    first such column in the stats; the columns before it match the oracle."""
    m, n = 6000, 40
    A = gi.gaussian(m, n, seed=23, dtype="fp32")
    A[:, 17] = A[:, 5]
    X = gi.to_float64(A, "fp32")
    rc, Q, R = (host_factor if path == "host" else device_factor)(h, A, "tf32x3")
    assert rc == 1
    assert h.stats()["first_breakdown_col"] == 17
    assert R[17, 17] == 0 and np.all(Q[:, 17] == 0)
    ref = oracle.rgs(X[:, :17], leaf=64)
    assert oracle.r_rel_error(R[:17, :17], ref.R) <= 1e-5


def test_non_finite_input_flagged(h):
    """A NaN in the input never yields a silently wrong factorization: the column's r_jj is not finite,
    so it is flagged (RGSQR_WARN_RANK_DEFICIENT) at or before the NaN's column."""
    A = gi.gaussian(4096, 32, seed=24, dtype="fp32")
    A[100, 9] = np.nan
    rc, Q, R = device_factor(h, A, "tf32")
    assert rc == 1
    assert 0 <= h.stats()["first_breakdown_col"] <= 9


def test_in_place_q_aliases_a_ragged(h):
    """Q_out == A_host (in place) with a ragged m (staged through the zero-padded bounce buffers)."""
    m, n = 10001, 150
    lda = _lda(m, "fp16")
    A = np.zeros((lda, n), dtype=np.float16, order="F")
    A[:m] = gi.gaussian(m, n, seed=25, dtype="fp16")
    X = gi.to_float64(np.asfortranarray(A[:m]), "fp16")
    pad = A[m:].copy()
    R = np.zeros((n, n), dtype=np.float32, order="F")
    rc = h.factor(A, lda, m, n, A, R, precision="fp16")
    assert rc == 0
    check(X, gi.to_float64(np.asfortranarray(A[:m]), "fp16"), R.astype(np.float64), "fp16")
    assert np.array_equal(A[m:], pad)   # rows past m untouched


def test_distributed_context_ragged_host(h):
    """A one-rank distributed context (every row-sharded code path: NCCL R12 all-reduce, peer exchange words,
    round-0 all-reduce) on a ragged host problem equals the plain context bitwise."""
    from paper_conf_icpp_zhangw21_b200 import Handle
    m, n = 9001, 200
    A = gi.gaussian(m, n, seed=26, dtype="fp16")
    d = Handle(0, rank=0, nranks=1, unique_id=Handle.unique_id())
    out = []
    h.set_option("fuse_small", 0)   # (single-GPU-only fused bottom node: compare the same products)
    try:
        for hh in (h, d):
            # the automatic split-K factor and tile heights depend on free arena space, which the
            # rank-reduction buffers change: pin them so both contexts take the same plan (as
            # tests/test_gpu_dist.py::test_host_ooc_dist_equals_plain)
            hh.set_option("splitk", 2)
            hh.set_option("tile_rows_min", 2048)
            hh.set_option("tile_rows_max", 2048)
            out.append(host_factor(hh, A, "fp16", budget=6 << 20))
            hh.set_option("splitk", 0)
            hh.set_option("tile_rows_min", 4096)
            hh.set_option("tile_rows_max", 16384)
    finally:
        d.close()
        h.set_option("fuse_small", 1)
    (rc1, Q1, R1), (rc2, Q2, R2) = out
    assert rc1 == 0 and rc2 == 0
    np.testing.assert_array_equal(Q1, Q2)
    np.testing.assert_array_equal(R1, R2)

"""GPU parity of the host-resident (out-of-core) factorization rgsqr_factor against the
oracle, across device budgets, reuse / serialize / blocked modes, plus the byte
counters against the paper's data-movement model (oracle/model.py)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

import oracle  # noqa: E402
from oracle import model  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402

MiB = 1 << 20
STOR = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32"}


@pytest.fixture()
def h():
    from paper_conf_icpp_zhangw21_b200 import Handle
    hd = Handle(0)
    yield hd
    hd.close()


def factor(h, A, prec, budget, **opts):
    m, n = A.shape
    for k, v in opts.items():
        h.set_option(k, v)
    Q = np.empty_like(A, order="F")
    R = np.full((n, n), np.nan, dtype=np.float32, order="F")
    rc = h.factor(A, m, m, n, Q, R, precision=prec, budget=budget)
    return rc, Q, R, h.stats()


@pytest.fixture(scope="module")
def gauss():
    A = gi.gaussian(16384, 1024, seed=7, dtype="fp16")
    X = gi.to_float64(A, "fp16")
    return A, X, oracle.rgs(X, leaf=64)


@pytest.mark.parametrize("budget_mib,reuse", [(0, 1), (80, 1), (40, 1), (28, 1), (28, 0), (20, 0), (20, 1), (12, 1), (12, 0)])
def test_ooc_gaussian_fp16(h, gauss, budget_mib, reuse):
    A, X, ref = gauss
    rc, Q, R, st = factor(h, A, "fp16", budget_mib * MiB, reuse=reuse)
    assert rc == 0
    Rg = R.astype(np.float64)
    assert oracle.is_upper_triangular(Rg)
    be = oracle.backward_error(X, gi.to_float64(Q, "fp16"), Rg)
    re = oracle.r_rel_error(Rg, ref.R)
    assert be < 5e-3 and re < 5e-3, (be, re, st)
    if budget_mib:
        assert st["arena_bytes"] + st["ctx_device_bytes"] <= budget_mib * MiB
    if 0 < budget_mib < 44:            # the whole 32 MiB matrix + workspace needs ~44.5 MiB
        assert st["n_ooc_nodes"] >= 1
    assert st["h2d_matrix_bytes"] >= A.nbytes and st["d2h_matrix_bytes"] >= A.nbytes


@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32"])
@pytest.mark.parametrize("budget_mib,reuse,algo", [(12, 1, 0), (20, 0, 0), (40, 1, 1), (40, 0, 1)])
def test_ooc_exact_dyadic(h, prec, budget_mib, reuse, algo):
    """Exact-dyadic input: every intermediate is exact, so any tile plan / budget /
    algorithm must return R == R0 and Q == H bitwise."""
    m, n = 16384, 1024
    A64, R0 = gi.dyadic_mixed(m, n, seed=5)
    A = gi.to_storage(A64, STOR[prec])
    budget = budget_mib * MiB * (2 if prec == "tf32" else 1)
    rc, Q, R, st = factor(h, A, prec, budget, reuse=reuse, algo=algo, block_cols=256)
    assert rc == 0
    np.testing.assert_array_equal(R.astype(np.float64), R0)
    np.testing.assert_array_equal(gi.to_float64(Q, STOR[prec]), gi.hadamard(m, n))


def test_serialized_equals_overlapped_bitwise(h, gauss):
    A = gauss[0]
    _, Q1, R1, st1 = factor(h, A, "fp16", 28 * MiB, serialize=0)
    _, Q2, R2, st2 = factor(h, A, "fp16", 28 * MiB, serialize=1)
    np.testing.assert_array_equal(R1, R2)
    np.testing.assert_array_equal(Q1, Q2)
    assert st1["h2d_bytes"] == st2["h2d_bytes"]


def test_in_place_q_aliases_a(h):
    m, n = 8192, 512
    A = gi.gaussian(m, n, seed=3, dtype="bf16")
    X = gi.to_float64(A, "bf16")
    R = np.zeros((n, n), dtype=np.float32, order="F")
    rc = h.factor(A, m, m, n, A, R, precision="bf16", budget=12 * MiB)      # Q_out = A_host
    assert rc == 0
    assert oracle.backward_error(X, gi.to_float64(A, "bf16"), R.astype(np.float64)) < 5e-3


def test_noreuse_bytes_match_recursive_model(h, gauss):
    """Budget 20 MiB at 16384 x 1024 fp16: in-core nodes of 256 columns (8 MiB + workspace),
    two OOC levels.  Without reuse the schedule moves exactly the model's words."""
    A = gauss[0]
    m, n = A.shape
    _, _, _, st = factor(h, A, "fp16", 20 * MiB, reuse=0)
    w = model.recursive_noreuse_split_words(m, n, 256)
    assert st["h2d_matrix_bytes"] == 2 * w["h2d_matrix"]
    assert st["d2h_matrix_bytes"] == 2 * w["d2h_matrix"]
    assert st["d2h_r_bytes"] == 4 * w["d2h_r"]


def test_noreuse_bytes_match_blocked_model(h, gauss):
    A = gauss[0]
    m, n = A.shape
    _, _, _, st = factor(h, A, "fp16", 40 * MiB, reuse=0, algo=1, block_cols=256)
    w = model.blocked_noreuse_split_words(m, n, 256)
    assert st["h2d_matrix_bytes"] == 2 * w["h2d_matrix"]
    assert st["d2h_matrix_bytes"] == 2 * w["d2h_matrix"]
    assert st["d2h_r_bytes"] == 4 * w["d2h_r"]


def test_reuse_moves_fewer_bytes_and_recursive_beats_blocked(h, gauss):
    A = gauss[0]
    _, _, _, s_reuse = factor(h, A, "fp16", 28 * MiB, reuse=1)
    _, _, _, s_plain = factor(h, A, "fp16", 28 * MiB, reuse=0)
    _, _, _, s_blk = factor(h, A, "fp16", 28 * MiB, reuse=0, algo=1, block_cols=128)
    assert s_reuse["h2d_bytes"] < s_plain["h2d_bytes"]
    assert s_plain["h2d_bytes"] < s_blk["h2d_bytes"]          # PAPER.md:155, Table 3


def test_budget_too_small(h):
    from paper_conf_icpp_zhangw21_b200 import RgsqrError
    A = gi.gaussian(16384, 256, seed=1, dtype="fp16")
    with pytest.raises(RgsqrError) as e:
        factor(h, A, "fp16", 1 * MiB)
    assert e.value.status == -2


def test_zero_column_warning(h):
    m, n = 8192, 256
    A = gi.gaussian(m, n, seed=2, dtype="fp16")
    A[:, 100] = 0
    rc, Q, R, st = factor(h, A, "fp16", 8 * MiB)
    assert rc == 1 and st["first_breakdown_col"] == 100
    assert R[100, 100] == 0


def test_ooc_tf32x3(h):
    m, n = 16384, 512
    A = gi.gaussian(m, n, seed=9, dtype="fp32")
    X = gi.to_float64(A, "fp32")
    rc, Q, R, st = factor(h, A, "tf32x3", 40 * MiB)
    assert rc == 0 and st["n_ooc_nodes"] >= 1
    Rg = R.astype(np.float64)
    assert oracle.backward_error(X, Q.astype(np.float64), Rg) <= 1e-5
    assert oracle.r_rel_error(Rg, oracle.rgs(X, leaf=64).R) <= 1e-5


@pytest.mark.parametrize("split_pct", [38, 62])
def test_ooc_split_ratio_ablation(h, gauss, split_pct):
    """RGSQR_OPT_SPLIT_PCT moves the split of out-of-core nodes away from the paper's halves
    (PAPER.md:115); the factorization is the same up to rounding order."""
    A, X, ref = gauss
    rc, Q, R, st = factor(h, A, "fp16", 20 * MiB, split_pct=split_pct)
    h.set_option("split_pct", 50)
    assert rc == 0 and st["n_ooc_nodes"] >= 1
    Rg = R.astype(np.float64)
    assert oracle.is_upper_triangular(Rg)
    assert oracle.backward_error(X, gi.to_float64(Q, "fp16"), Rg) < 5e-3
    assert oracle.r_rel_error(Rg, ref.R) < 5e-3


@pytest.mark.parametrize("prec,lda_pad", [("fp16", 8), ("bf16", 120), ("tf32", 4)])
def test_host_path_lda_greater_than_m(h, prec, lda_pad):
    """lda > m (LAPACK convention, include/rgsqr.h): A and Q live in a taller host buffer; the
    rows [m, lda) of Q_out must not be touched, and the result equals the lda = m run bitwise
    (same tiles, same kernels), out-of-core under a small budget."""
    st = STOR[prec]
    m, n = 8192, 512
    lda = m + lda_pad
    A = gi.gaussian(m, n, seed=21, dtype=st)
    big = np.zeros((lda, n), dtype=A.dtype, order="F")
    big[:m] = A
    Qb = np.full_like(big, 7, order="F")
    Rb = np.full((n, n), np.nan, dtype=np.float32, order="F")
    budget = 6 * MiB if st != "fp32" else 12 * MiB
    rc = h.factor(big, lda, m, n, Qb, Rb, precision=prec, budget=budget)
    assert rc == 0 and h.stats()["n_ooc_nodes"] >= 1
    assert np.all(Qb[m:] == 7)
    rc, Q, R, _ = factor(h, np.asfortranarray(A), prec, budget)
    np.testing.assert_array_equal(Rb, R)
    np.testing.assert_array_equal(Qb[:m], Q)


@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32"])
@pytest.mark.parametrize("budget_mib", [34, 38, 40])
def test_colchunk_node_vs_streamed_node(h, prec, budget_mib):
    """Column-chunked OOC node (RGSQR_OPT_COLCHUNK, R26; PAPER.md:231-233 cross-operation
    overlap): the right child starts while A2's later columns are in flight, the tail that does not
    fit beside Q1 is projected from the host first.  Same factorization as the row-tile streamed
    node (Eq. 2): both against the oracle, and against each other."""
    st = STOR[prec]
    m, n = 16384, 1024
    A = gi.gaussian(m, n, seed=31, dtype=st)
    X = gi.to_float64(A, st)
    ref = oracle.rgs(X, leaf=64)
    budget = budget_mib * MiB * (2 if st == "fp32" else 1)
    out = {}
    for cc in (1, 0):
        # 2 MiB upload chunks: 64-column pieces at this height, so the first-projection phase
        # and the chunked pieces of the column-chunked node all occur (32 MiB would be 1 chunk)
        rc, Q, R, stt = factor(h, A, prec, budget, colchunk=cc, chunk_mib=2)
        assert rc == 0 and stt["n_ooc_nodes"] >= 1 and stt["arena_bytes"] + stt["ctx_device_bytes"] <= budget
        if cc:
            assert stt["n_colchunk_nodes"] >= 1, stt
        else:
            assert stt["n_colchunk_nodes"] == 0
        Rg = R.astype(np.float64)
        assert oracle.is_upper_triangular(Rg)
        be = oracle.backward_error(X, gi.to_float64(Q, st), Rg)
        re = oracle.r_rel_error(Rg, ref.R)
        assert be < 5e-3 and re < 5e-3, (cc, be, re, stt)
        out[cc] = Rg
    h.set_option("colchunk", 1)
    h.set_option("chunk_mib", 32)
    assert oracle.r_rel_error(out[1], out[0]) < 2e-3


@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32"])
def test_colchunk_node_dyadic_bitwise(h, prec):
    """Exact-dyadic input through the column-chunked node: R == R0 and Q == H
    bitwise, whatever the column split, the tail's host round trip and the chunked projections."""
    st = STOR[prec]
    m, n = 16384, 1024
    A64, R0 = gi.dyadic_mixed(m, n, seed=9)
    A = gi.to_storage(A64, st)
    for budget_mib, chunk in ((34, 32), (40, 2), (38, 1)):
        budget = budget_mib * MiB * (2 if st == "fp32" else 1)
        rc, Q, R, stt = factor(h, A, prec, budget, colchunk=1, chunk_mib=chunk)
        assert rc == 0 and stt["n_colchunk_nodes"] >= 1, stt
        np.testing.assert_array_equal(R.astype(np.float64), R0)
        np.testing.assert_array_equal(gi.to_float64(Q, st), gi.hadamard(m, n))
    h.set_option("chunk_mib", 32)


def test_colchunk_serialized_equals_overlapped(h):
    """Race check of the column-chunked node: one stream (RGSQR_OPT_SERIALIZE) == overlapped, bitwise."""
    A = gi.gaussian(16384, 1024, seed=33, dtype="fp16")
    _, Q1, R1, s1 = factor(h, A, "fp16", 40 * MiB, colchunk=1, serialize=1, chunk_mib=2)
    _, Q2, R2, s2 = factor(h, A, "fp16", 40 * MiB, colchunk=1, serialize=0, chunk_mib=2)
    h.set_option("chunk_mib", 32)
    assert s1["n_colchunk_nodes"] >= 1 and s2["n_colchunk_nodes"] >= 1
    np.testing.assert_array_equal(R1, R2)
    np.testing.assert_array_equal(Q1, Q2)


def test_host_alloc_numa_buffers(h):
    """rgsqr_host_alloc: NUMA-placed, page-locked buffers (include/rgsqr.h) used as A / Q / R of the
    out-of-core path; results equal those from pageable numpy buffers; freeing twice is an error."""
    import ctypes
    from paper_conf_icpp_zhangw21_b200 import RgsqrError
    m, n = 8192, 512
    A = gi.gaussian(m, n, seed=41, dtype="fp16")
    nb = A.nbytes
    pa, pq, pr = h.host_alloc(nb), h.host_alloc(nb), h.host_alloc(n * n * 4)
    np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(pa))[:] = A.reshape(-1, order="F").view(np.uint8)
    assert h.factor(pa, m, m, n, pq, pr, precision="fp16", budget=6 * MiB) == 0
    Qp = np.ctypeslib.as_array((ctypes.c_uint16 * (m * n)).from_address(pq)).view(np.float16).reshape((m, n), order="F")
    Rp = np.ctypeslib.as_array((ctypes.c_float * (n * n)).from_address(pr)).reshape((n, n), order="F")
    rc, Q, R, _ = factor(h, A, "fp16", 6 * MiB)
    np.testing.assert_array_equal(Rp, R)
    np.testing.assert_array_equal(Qp, Q)
    for p_ in (pa, pq, pr):
        h.host_free(p_)
    with pytest.raises(RgsqrError):
        h.host_free(pa)


@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32"])
def test_fused_blocked_algorithm(h, prec):
    """RGSQR_OPT_ALGO = 2 (fused blocked, SURVEY.md 8(f) f1 honesty variant): the blocked loop of
    PAPER.md:113 with the panel resident and the trailing matrix read and written once per panel in
    column blocks.  Against the oracle, exact-dyadic bitwise, and its byte count: each direction moves
    m s sum_i (n - i b) = m n s (k + 1) / 2 for k = n / b panels."""
    st = STOR[prec]
    m, n, b = 16384, 1024, 256
    s = 4 if st == "fp32" else 2
    budget = (24 if s == 2 else 48) * MiB
    A = gi.gaussian(m, n, seed=51, dtype=st)
    X = gi.to_float64(A, st)
    rc, Q, R, stt = factor(h, A, prec, budget, algo=2, block_cols=b)
    assert rc == 0
    Rg = R.astype(np.float64)
    ref = oracle.rgs(X, leaf=64)
    assert oracle.backward_error(X, gi.to_float64(Q, st), Rg) < 5e-3
    assert oracle.r_rel_error(Rg, ref.R) < 5e-3
    k = n // b
    assert stt["h2d_matrix_bytes"] == m * n * s * (k + 1) // 2
    assert stt["d2h_matrix_bytes"] == m * n * s * (k + 1) // 2
    A64, R0 = gi.dyadic_mixed(m, n, seed=52)
    rc, Q, R, _ = factor(h, gi.to_storage(A64, st), prec, budget, algo=2, block_cols=b)
    np.testing.assert_array_equal(R.astype(np.float64), R0)
    np.testing.assert_array_equal(gi.to_float64(Q, st), gi.hadamard(m, n))

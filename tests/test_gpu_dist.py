"""The row-sharded (distributed) code paths on one GPU: a distributed context with one rank
runs the round-0 NCCL allreduce, the R12 rank reduction and the .sys exchange of the leaf.
Sums over one rank are identities, so results must be BITWISE equal to the plain context."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from tests.gpu_util import to_dev, from_dev  # noqa: E402

MiB = 1 << 20
STOR = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32"}


@pytest.fixture(scope="module")
def handles():
    from paper_conf_icpp_zhangw21_b200 import Handle
    plain = Handle(0)
    # the fused bottom-node kernel is a single-GPU path (its R12 reduction cannot include other
    # ranks); compare against the plain context running the same separate products
    plain.set_option("fuse_small", 0)
    dist = Handle(0, rank=0, nranks=1, unique_id=Handle.unique_id())
    yield plain, dist
    dist.close()
    plain.close()


def _dev_factor(h, A, prec, m, n):
    st = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32", "tf32x3": "fp32"}[prec]
    Ad = to_dev(A, st)
    R = torch.empty((n, n), dtype=torch.float32, device="cuda")
    rc = h.factor_device(Ad, m, m, n, Ad, R, precision=prec)
    return rc, from_dev(Ad), R.cpu().numpy().T


@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32", "tf32x3"])
def test_device_dist_equals_plain(handles, prec):
    """(tf32x3: the plain context's nodes share one Q1 hi / lo split between both products, op_node_x3;
    the distributed context runs the separate inner / outer products -- bitwise equal, split-K pinned
    because the automatic factor follows the free arena, which the rank-reduction buffer changes)"""
    plain, dist = handles
    m, n = 16384, 512
    A = gi.gaussian(m, n, seed=11, dtype={"fp16": "fp16", "bf16": "bf16", "tf32": "fp32", "tf32x3": "fp32"}[prec])
    sk = 4 if prec == "tf32x3" else 0
    plain.set_option("splitk", sk)
    dist.set_option("splitk", sk)
    try:
        _, Q1, R1 = _dev_factor(plain, A, prec, m, n)
        _, Q2, R2 = _dev_factor(dist, A, prec, m, n)
    finally:
        plain.set_option("splitk", 0)
        dist.set_option("splitk", 0)
    np.testing.assert_array_equal(R1, R2)
    np.testing.assert_array_equal(Q1, Q2)


def test_host_ooc_dist_equals_plain(handles):
    plain, dist = handles
    m, n = 16384, 1024
    A = gi.gaussian(m, n, seed=12, dtype="fp16")
    out = []
    for h in (plain, dist):
        # the automatic split-K factor depends on free arena space, which the rank-reduction
        # buffer changes; pin it so both runs sum the same partials in the same order
        # (and the in-core threshold / ring tile height, so both take the same plan)
        h.set_option("splitk", 2)
        h.set_option("tile_rows_min", 2048)
        h.set_option("tile_rows_max", 2048)
        Q = np.empty_like(A, order="F")
        R = np.zeros((n, n), dtype=np.float32, order="F")
        assert h.factor(A, m, m, n, Q, R, precision="fp16", budget=28 * MiB) == 0
        assert h.stats()["n_ooc_nodes"] == 1
        h.set_option("splitk", 0)
        h.set_option("tile_rows_min", 4096)
        h.set_option("tile_rows_max", 16384)
        out.append((Q, R))
    np.testing.assert_array_equal(out[0][1], out[1][1])
    np.testing.assert_array_equal(out[0][0], out[1][0])


def test_dist_exact_dyadic(handles):
    _, dist = handles
    m, n = 16384, 768
    A64, R0 = gi.dyadic_mixed(m, n, seed=8)
    A = gi.to_storage(A64, "bf16")
    Q = np.empty_like(A, order="F")
    R = np.zeros((n, n), dtype=np.float32, order="F")
    assert dist.factor(A, m, m, n, Q, R, precision="bf16", budget=16 * MiB) == 0
    np.testing.assert_array_equal(R.astype(np.float64), R0)


def test_repeated_launches_keep_exchange_state(handles):
    """The leaf's exchange words are never reset; many launches in a row must stay exact."""
    _, dist = handles
    m, n = 4096, 64
    H = gi.hadamard(m, n)
    for _ in range(5):
        Pd = to_dev(gi.to_storage(H, "fp16"), "fp16")
        R = torch.zeros((n, n), dtype=torch.float32, device="cuda")
        dist.op_leaf(Pd, m, m, n, R, n, precision="fp16")
        np.testing.assert_array_equal(R.cpu().numpy().T, np.eye(n))


# ---- virtual row shards (RGSQR_OPT_VSHARDS): the multi-GPU arithmetic on one GPU ----------------
@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32"])
@pytest.mark.parametrize("p", [2, 4, 8])
def test_vshards_dyadic_bitwise_equal_single(prec, p):
    """p row shards on one GPU: every R12 as p local products summed in shard order, every leaf's
    round-0 vector as p local vectors summed in shard order (the NCCL allreduces of a p-GPU run,
    DESIGN.md 8; PAPER.md:171-173 row-local structure).  Exact-dyadic input: R == R0
    and Q == H bitwise for every p, hence bitwise equal to the single-GPU result."""
    from paper_conf_icpp_zhangw21_b200 import Handle
    st = STOR[prec]
    m, n = 65536, 512
    A64, R0 = gi.dyadic_mixed(m, n, seed=13)
    A = gi.to_storage(A64, st)
    h = Handle(0)
    h.set_option("vshards", p)
    Ad = to_dev(A, st)
    R = torch.empty((n, n), dtype=torch.float32, device="cuda")
    rc = h.factor_device(Ad, m, m, n, Ad, R, precision=prec)
    assert rc == 0
    np.testing.assert_array_equal(R.cpu().numpy().T.astype(np.float64), R0)
    np.testing.assert_array_equal(from_dev(Ad), gi.hadamard(m, n))
    h.close()


@pytest.mark.parametrize("prec", ["fp16", "tf32"])
def test_vshards_gaussian_vs_single_and_oracle(prec):
    from paper_conf_icpp_zhangw21_b200 import Handle
    st = STOR[prec]
    m, n = 16384, 1024
    A = gi.gaussian(m, n, seed=17, dtype=st)
    X = gi.to_float64(A, st)
    ref = oracle.rgs(X, leaf=64)
    h = Handle(0)
    out = {}
    for p in (1, 4):
        h.set_option("vshards", p)
        Ad = to_dev(A, st)
        R = torch.empty((n, n), dtype=torch.float32, device="cuda")
        assert h.factor_device(Ad, m, m, n, Ad, R, precision=prec) == 0
        Rn = R.cpu().numpy().T.astype(np.float64)
        Q = from_dev(Ad)
        assert oracle.backward_error(X, Q, Rn) < 5e-3
        assert oracle.r_rel_error(Rn, ref.R) < 5e-3
        out[p] = Rn
    assert oracle.r_rel_error(out[4], out[1]) < 2e-3
    h.close()


def test_vshards_rejects_unequal_shards():
    from paper_conf_icpp_zhangw21_b200 import Handle, RgsqrError
    h = Handle(0)
    h.set_option("vshards", 3)
    A = gi.gaussian(4096, 64, seed=1, dtype="fp16")
    Ad = to_dev(A, "fp16")
    R = torch.empty((64, 64), dtype=torch.float32, device="cuda")
    with pytest.raises(RgsqrError) as e:
        h.factor_device(Ad, 4096, 4096, 64, Ad, R, precision="fp16")
    assert e.value.status == -5
    h.close()


def test_host_colchunk_dist_equals_plain(handles):
    """The column-chunked out-of-core node (R26) in a distributed context: its tail, phase-A
    and piece-wise projections reduce R12 across ranks (ncclAllReduce).  The distributed context
    reserves the reduction buffers, so its plan (tail width) can differ from the plain one: Gaussian
    results agree to rounding, exact-dyadic results are bitwise R0 / H for both."""
    plain, dist = handles
    m, n = 16384, 1024
    A = gi.gaussian(m, n, seed=14, dtype="fp16")
    A64, R0 = gi.dyadic_mixed(m, n, seed=15)
    Ad = gi.to_storage(A64, "fp16")
    out = []
    for h in (plain, dist):
        h.set_option("chunk_mib", 2)
        Q = np.empty_like(A, order="F")
        R = np.zeros((n, n), dtype=np.float32, order="F")
        assert h.factor(A, m, m, n, Q, R, precision="fp16", budget=40 * MiB) == 0
        st = h.stats()
        assert st["n_colchunk_nodes"] == 1, (h is plain, {k: st[k] for k in ("h2d_bytes", "n_ooc_nodes", "arena_bytes", "ctx_device_bytes") if k in st}, st)
        out.append(R.astype(np.float64))
        Qd = np.empty_like(Ad, order="F")
        Rd = np.zeros((n, n), dtype=np.float32, order="F")
        assert h.factor(Ad, m, m, n, Qd, Rd, precision="fp16", budget=40 * MiB) == 0
        assert h.stats()["n_colchunk_nodes"] == 1
        np.testing.assert_array_equal(Rd.astype(np.float64), R0)
        np.testing.assert_array_equal(gi.to_float64(Qd, "fp16"), gi.hadamard(m, n))
        h.set_option("chunk_mib", 32)
    assert np.linalg.norm(out[0] - out[1]) / np.linalg.norm(out[0]) < 2e-3


def test_budget_agreement_follows_each_call(handles):
    """The distributed budget agreement (ncclAllReduce of the shape / budget words) must see THIS
    call's budget: a smaller budget in the previous call must not leak into the next plan."""
    _, dist = handles
    m, n = 8192, 256
    A = gi.gaussian(m, n, seed=21, dtype="fp16")
    for b in (12, 40, 10, 64, 12):
        Q = np.empty_like(A, order="F")
        R = np.zeros((n, n), dtype=np.float32, order="F")
        assert dist.factor(A, m, m, n, Q, R, precision="fp16", budget=b * MiB) == 0
        st = dist.stats()
        assert st["arena_bytes"] == b * MiB - st["ctx_device_bytes"], (b, st["arena_bytes"])


def test_dist_tall_panel_equals_plain(handles):
    """Tall leaf panels (> 2048 rows per CTA, leaf.cu NR = 0) through the row-sharded code paths (round-0-only
    launch + all-reduce, peer exchange words): bitwise equal to the plain context."""
    plain, dist = handles
    m, n = 600000, 48
    A = gi.gaussian(m, n, seed=13, dtype="fp16")
    for h in (plain, dist):
        h.set_option("splitk", 8)
    try:
        _, Q1, R1 = _dev_factor(plain, A, "fp16", m, n)
        _, Q2, R2 = _dev_factor(dist, A, "fp16", m, n)
    finally:
        for h in (plain, dist):
            h.set_option("splitk", 0)
    np.testing.assert_array_equal(R1, R2)
    np.testing.assert_array_equal(Q1, Q2)

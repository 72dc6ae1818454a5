"""GPU parity of the three hot-path kernels (C ABI rgsqr_op_*) against the CPU oracle /
fp64 library products of the same stored operands."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from tests.gpu_util import to_dev, from_dev, TORCH_DT  # noqa: E402

PRECS = [("fp16", "fp16"), ("bf16", "bf16"), ("tf32", "fp32")]


@pytest.fixture(scope="module")
def h():
    from paper_conf_icpp_zhangw21_b200 import Handle
    hd = Handle(0)
    yield hd
    hd.close()


def _rand(m, n, seed, storage):
    return gi.gaussian(m, n, seed=seed, dtype=storage)


@pytest.mark.parametrize("prec,storage", PRECS)
@pytest.mark.parametrize("m,w1,w2,splitk", [(8192, 192, 320, 0), (2048, 1024, 768, 1), (1000, 64, 40, 0),
                                            (4096, 130, 257, 3)])
def test_inner_product(h, prec, storage, m, w1, w2, splitk):
    A = _rand(m, w1 + w2, 11, storage)
    Ad = to_dev(A, storage)
    X = gi.to_float64(A, storage)
    ref = X[:, :w1].T @ X[:, w1:]
    R = torch.zeros((w2, w1), dtype=torch.float32, device="cuda")       # col-major w1 x w2
    Rop = torch.zeros((w2, w1), dtype=TORCH_DT[storage], device="cuda")
    h.set_option("splitk", splitk)
    try:
        h.op_inner(Ad, m, Ad[w1:], m, m, w1, w2, R, w1, Rop, accumulate=False, precision=prec)
        got = R.cpu().numpy().T
        scale = np.sqrt(m) * 4
        tol = (2e-5 if storage != "fp32" else 2e-3) * scale
        np.testing.assert_allclose(got, ref, rtol=0, atol=tol)
        # accumulate: R += Q1^T A2 again
        h.op_inner(Ad, m, Ad[w1:], m, m, w1, w2, R, w1, Rop, accumulate=True, precision=prec)
        np.testing.assert_allclose(R.cpu().numpy().T, 2 * ref, rtol=0, atol=2 * tol)
        opv = Rop.to(torch.float32).cpu().numpy().T
        np.testing.assert_allclose(opv, R.cpu().numpy().T, rtol=1e-2 if storage == "bf16" else 1e-3, atol=1e-3)
    finally:
        h.set_option("splitk", 0)


@pytest.mark.parametrize("prec,storage", PRECS)
@pytest.mark.parametrize("m,w1,w2", [(4096, 192, 320), (1000, 64, 40), (33000, 256, 256), (640, 72, 300)])
def test_outer_product(h, prec, storage, m, w1, w2):
    Q = _rand(m, w1, 21, storage)
    A2 = _rand(m, w2, 22, storage)
    R12 = gi.to_storage(np.random.default_rng(3).standard_normal((w1, w2)) / np.sqrt(w1), storage)
    Qd, A2d, Rd = to_dev(Q, storage), to_dev(A2, storage), to_dev(R12, storage)
    Xq, Xa, Xr = (gi.to_float64(x, storage) for x in (Q, A2, R12))
    ref = Xa - Xq @ Xr
    h.op_outer(Qd, m, Rd, w1, A2d, m, m, w1, w2, precision=prec)
    got = from_dev(A2d)
    ulp = {"fp16": 2 ** -11, "bf16": 2 ** -8, "fp32": 2 ** -11}[storage]   # tf32 operands: 2^-11
    tol = 4 * ulp * (np.abs(ref) + np.abs(Xq) @ np.abs(Xr)) + 1e-6
    assert np.all(np.abs(got - ref) <= tol), float(np.max(np.abs(got - ref) / tol))


@pytest.mark.parametrize("prec,storage", PRECS)
# (400000, 15), (600000, 9), (1048576, 4): more than LEAF_MAX_RP = 2048 rows per CTA -> the tall leaf
# (row state in shared memory, kernels.h LEAF_MAX_RP_TALL); widths are the widest that fit on chip
@pytest.mark.parametrize("m,w", [(20000, 64), (4096, 32), (1000, 7), (300, 64), (65536, 64), (131072, 48), (262144, 24),
                                 (400000, 15), (600000, 9), (1048576, 4)])
def test_leaf_cgs(h, prec, storage, m, w):
    A = _rand(m, w, 31, storage)
    X = gi.to_float64(A, storage)
    ref = oracle.cgs(X)
    Pd = to_dev(A, storage)
    R = torch.zeros((w, w), dtype=torch.float32, device="cuda")
    rc, brk = h.op_leaf(Pd, m, m, w, R, w, precision=prec)
    assert rc == 0 and brk == -1
    Rg = R.cpu().numpy().T.astype(np.float64)
    Qg = from_dev(Pd)
    assert oracle.is_upper_triangular(Rg)
    u = {"fp16": 2 ** -11, "bf16": 2 ** -8, "fp32": 2 ** -24}[storage]
    assert oracle.r_rel_error(Rg, ref.R) < 50 * 2 ** -24 * np.sqrt(m) + 1e-6
    assert np.max(np.abs(Qg - ref.Q)) < 4 * u + 1e-5
    assert oracle.backward_error(X, Qg, Rg) < 4 * u


def test_leaf_exact_hadamard(h):
    m, w = 4096, 64
    H = gi.hadamard(m, w)
    Pd = to_dev(gi.to_storage(H, "fp16"), "fp16")
    R = torch.zeros((w, w), dtype=torch.float32, device="cuda")
    h.op_leaf(Pd, m, m, w, R, w, precision="fp16")
    np.testing.assert_array_equal(R.cpu().numpy().T, np.eye(w))
    np.testing.assert_array_equal(from_dev(Pd), H)


def test_leaf_zero_column_breakdown(h):
    m, w = 5000, 16
    A = _rand(m, w, 5, "fp32")
    A[:, 9] = 0
    Pd = to_dev(A, "fp32")
    R = torch.zeros((w, w), dtype=torch.float32, device="cuda")
    rc, brk = h.op_leaf(Pd, m, m, w, R, w, precision="tf32")
    assert rc == 1 and brk == 9
    assert R[9, 9].item() == 0.0

"""GPU parity of the standalone out-of-core GEMMs (rgsqr_ooc_inner / rgsqr_ooc_outer; the paper's
Tables 1/2 operations) against fp64 products of the stored operands,
for both tilings (recursive: Figs. 3/5, blocking: Figs. 4/6), under budgets that force many tiles.

Bounds: the tensor cores multiply the stored operands exactly (fp16 / bf16) or after tf32 rounding
(2^-11 relative, R5) and accumulate in fp32, so |dR12_ij| <= c (|Q1|^T |A2|)_ij with c = 1e-4
(16-bit) or 2e-3 (tf32); the outer product uses R12 rounded to the operand type (R9) and stores
A2' rounded RN: |dA2'_ij| <= u_s |A2'_ij| + c (|Q1| |R12op|)_ij."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

import rgsqr_inputs as gi  # noqa: E402

MiB = 1 << 20
STOR = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32"}
U = {"fp16": 2.0 ** -11, "bf16": 2.0 ** -8, "tf32": 2.0 ** -24}
C = {"fp16": 1e-4, "bf16": 1e-4, "tf32": 2e-3}


@pytest.fixture()
def h():
    from paper_conf_icpp_zhangw21_b200 import Handle
    hd = Handle(0)
    yield hd
    hd.close()


def _ops(prec, m, w1, w2, seed):
    st = STOR[prec]
    Q = gi.gaussian(m, w1, seed=seed, dtype=st)
    A = gi.gaussian(m, w2, seed=seed + 1, dtype=st)
    return st, Q, A, gi.to_float64(Q, st), gi.to_float64(A, st)


@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32"])
@pytest.mark.parametrize("tiling,block", [(0, 2048), (0, 0), (1, 128), (1, 200)])
def test_ooc_inner(h, prec, tiling, block):
    m, w1, w2 = 20000, 384, 520
    st, Q, A, Xq, Xa = _ops(prec, m, w1, w2, 3)
    R = np.full((w1, w2), np.nan, dtype=np.float32, order="F")
    budget = 56 * MiB * (2 if st == "fp32" else 1)
    h.ooc_inner(Q, m, A, m, m, w1, w2, R, w1, precision=prec, tiling=tiling, block=block, budget=budget)
    ref = Xq.T @ Xa
    bound = C[prec] * (np.abs(Xq).T @ np.abs(Xa))
    assert np.all(np.abs(R - ref) <= bound), np.max(np.abs(R - ref) / bound)
    s = h.stats()
    assert s["arena_bytes"] + s["ctx_device_bytes"] <= budget and s["h2d_bytes"] >= Q.nbytes + A.nbytes


@pytest.mark.parametrize("prec", ["fp16", "bf16", "tf32"])
@pytest.mark.parametrize("tiling,block", [(0, 2048), (0, 0), (1, 1024), (1, 4096)])
def test_ooc_outer(h, prec, tiling, block):
    m, w1, w2 = 20000, 256, 520
    st, Q, A, Xq, Xa = _ops(prec, m, w1, w2, 5)
    R = np.asfortranarray((np.random.default_rng(1).standard_normal((w1, w2)) / np.sqrt(w1)).astype(np.float32))
    Rop = gi.to_float64(gi.to_storage(R.astype(np.float64), st), st)     # R12 as the MMA operand (R9)
    A2 = np.array(A, order="F", copy=True)
    h.ooc_outer(Q, m, R, w1, A2, m, m, w1, w2, precision=prec, tiling=tiling, block=block,
                budget=48 * MiB * (2 if st == "fp32" else 1))
    ref = Xa - Xq @ Rop
    got = gi.to_float64(A2, st)
    bound = U[prec] * np.abs(ref) + C[prec] * (np.abs(Xq) @ np.abs(Rop)) + 1e-30
    assert np.all(np.abs(got - ref) <= bound), np.max(np.abs(got - ref) / bound)


def test_ooc_gemm_serialized_equals_overlapped(h):
    """Race check: one stream (the paper's "Synchronous" rows) == overlapped, bitwise."""
    m, w1, w2 = 20000, 256, 384
    st, Q, A, _, _ = _ops("fp16", m, w1, w2, 7)
    out = []
    for ser in (1, 0):
        h.set_option("serialize", ser)
        R = np.empty((w1, w2), dtype=np.float32, order="F")
        h.ooc_inner(Q, m, A, m, m, w1, w2, R, w1, precision="fp16", tiling=0, block=2048, budget=32 * MiB)
        A2 = np.array(A, order="F", copy=True)
        h.ooc_outer(Q, m, R, w1, A2, m, m, w1, w2, precision="fp16", tiling=0, block=2048, budget=32 * MiB)
        out.append((R, A2))
    np.testing.assert_array_equal(out[0][0], out[1][0])
    np.testing.assert_array_equal(out[0][1], out[1][1])


def test_ooc_gemm_budget_too_small(h):
    from paper_conf_icpp_zhangw21_b200 import RgsqrError
    m, w1, w2 = 20000, 256, 384
    st, Q, A, _, _ = _ops("fp16", m, w1, w2, 9)
    R = np.empty((w1, w2), dtype=np.float32, order="F")
    with pytest.raises(RgsqrError) as e:
        h.ooc_inner(Q, m, A, m, m, w1, w2, R, w1, precision="fp16", budget=1 * MiB)
    assert e.value.status == -2

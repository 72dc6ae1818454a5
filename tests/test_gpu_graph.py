"""CUDA-graph replay of whole factorizations (RGSQR_OPT_GRAPH, csrc/graph.cu, R30).

The replayed graph must compute exactly what the eager launches compute (the schedule is the same
sequence of kernels and copies), across repeated replays, interleaved eager calls (the grid-barrier
counters the launches bake are reset by the graph), arena reallocations and option changes."""
import ctypes

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from tests.gpu_util import to_dev, from_dev  # noqa: E402

MiB = 1 << 20


@pytest.fixture()
def h():
    from paper_conf_icpp_zhangw21_b200 import Handle
    hd = Handle(0)
    yield hd
    hd.close()


class Pinned:
    """A / Q / R in rgsqr_host_alloc buffers (page-locked: the host path may replay a graph)."""

    def __init__(self, h, A):
        self.h, (self.m, self.n) = h, A.shape
        self.dt = A.dtype
        nb = A.nbytes
        self.pa, self.pq, self.pr = h.host_alloc(nb), h.host_alloc(nb), h.host_alloc(self.n * self.n * 4)
        self.A = np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(self.pa))
        self.A[:] = A.reshape(-1, order="F").view(np.uint8)
        self.Q = np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(self.pq))
        self.R = np.ctypeslib.as_array((ctypes.c_uint8 * (self.n * self.n * 4)).from_address(self.pr))

    def factor(self, prec, budget):
        rc = self.h.factor(self.pa, self.m, self.m, self.n, self.pq, self.pr, precision=prec, budget=budget)
        Q = self.Q.copy().view(self.dt).reshape((self.m, self.n), order="F")
        R = self.R.copy().view(np.float32).reshape((self.n, self.n), order="F")
        return rc, Q, R, self.h.stats()

    def free(self):
        for p in (self.pa, self.pq, self.pr):
            self.h.host_free(p)


@pytest.mark.parametrize("prec,budget_mib", [("fp16", 36), ("fp16", 80), ("bf16", 24), ("tf32", 64)])
def test_host_graph_replay_bitwise_equals_eager(h, prec, budget_mib):
    m, n = 16384, 1024
    st = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32"}[prec]
    A = gi.gaussian(m, n, seed=61, dtype=st)
    P = Pinned(h, A)
    h.set_option("graph", 0)
    rc, Q0, R0, s0 = P.factor(prec, budget_mib * MiB)
    assert rc == 0 and s0["graph_replay"] == 0
    h.set_option("graph", 1)
    for it in range(3):   # capture + launch, then two replays
        rc, Q1, R1, s1 = P.factor(prec, budget_mib * MiB)
        assert rc == 0
        assert s1["graph_replay"] == 1
        assert s1["graph_captures"] == 1, s1["graph_captures"]
        np.testing.assert_array_equal(R1, R0)
        np.testing.assert_array_equal(Q1, Q0)
        # the captured schedule's counters are reported on every replay
        for k in ("h2d_bytes", "d2h_bytes", "n_leaf_launches", "n_tn_launches", "n_nn_launches", "n_ooc_nodes",
                  "n_colchunk_nodes"):
            assert s1[k] == s0[k], k
    X = gi.to_float64(A, st)
    assert oracle.backward_error(X, gi.to_float64(Q1, st), R1.astype(np.float64)) < 5e-3
    P.free()


def test_host_graph_exact_dyadic(h):
    """Exact-dyadic input: every replay gives R == R0 and Q == H bitwise."""
    m, n = 16384, 1024
    A64, Rref = gi.dyadic_mixed(m, n, seed=62)
    A = gi.to_storage(A64, "fp16")
    P = Pinned(h, A)
    for _ in range(3):
        rc, Q, R, s = P.factor("fp16", 36 * MiB)
        assert rc == 0 and s["graph_replay"] == 1
        np.testing.assert_array_equal(R.astype(np.float64), Rref)
        np.testing.assert_array_equal(gi.to_float64(Q, "fp16"), gi.hadamard(m, n))
    P.free()


def test_graph_interleaved_with_eager_calls(h):
    """Replays interleaved with eager calls that use the same grid-barrier counters (pageable
    buffers -> eager host path; a device call with another shape -> its own graph)."""
    m, n = 16384, 512
    A = gi.gaussian(m, n, seed=63, dtype="fp16")
    P = Pinned(h, A)
    rc, Qg, Rg, _ = P.factor("fp16", 20 * MiB)
    assert rc == 0
    B = gi.gaussian(8192, 256, seed=64, dtype="fp16")
    XB = gi.to_float64(B, "fp16")
    for it in range(3):
        Qe = np.empty_like(B, order="F")
        Re = np.zeros((256, 256), dtype=np.float32, order="F")
        assert h.factor(B, 8192, 8192, 256, Qe, Re, precision="fp16", budget=8 * MiB) == 0
        assert h.stats()["graph_replay"] == 0          # (pageable numpy buffers: eager)
        assert oracle.backward_error(XB, gi.to_float64(Qe, "fp16"), Re.astype(np.float64)) < 5e-3
        Ad = to_dev(B, "fp16")
        Rd = torch.empty((256, 256), dtype=torch.float32, device="cuda")
        assert h.factor_device(Ad, 8192, 8192, 256, Ad, Rd, precision="fp16") == 0
        Rdn = Rd.cpu().numpy().T.astype(np.float64)
        assert oracle.backward_error(XB, from_dev(Ad), Rdn) < 5e-3
        assert oracle.r_rel_error(Rdn, Re.astype(np.float64)) < 2e-3
        rc, Q, R, s = P.factor("fp16", 20 * MiB)
        assert rc == 0 and s["graph_replay"] == 1
        np.testing.assert_array_equal(R, Rg)
        np.testing.assert_array_equal(Q, Qg)
    P.free()


def test_graph_recaptured_after_arena_and_option_changes(h):
    m, n = 16384, 512
    A = gi.gaussian(m, n, seed=65, dtype="fp16")
    P = Pinned(h, A)
    outs = {}
    for budget, leaf in ((20, 64), (200, 64), (20, 64), (20, 32), (20, 64)):
        h.set_option("leaf_width", leaf)
        rc, Q, R, s = P.factor("fp16", budget * MiB)
        assert rc == 0 and s["graph_replay"] == 1
        key = (budget, leaf)
        if key in outs:
            np.testing.assert_array_equal(R, outs[key][1])
            np.testing.assert_array_equal(Q, outs[key][0])
        outs[key] = (Q, R)
    # 20 -> 200 MiB reallocates the arena (captured graphs are dropped): 20/64 is captured twice
    assert h.stats()["graph_captures"] == 4
    h.set_option("leaf_width", 64)
    P.free()


def test_device_graph_replay_bitwise_equals_eager(h):
    m, n = 32768, 1024
    A = gi.gaussian(m, n, seed=66, dtype="fp16")
    outs = []
    for g in (0, 1, 1, 1):
        h.set_option("graph", g)
        Ad = to_dev(A, "fp16")
        R = torch.empty((n, n), dtype=torch.float32, device="cuda")
        assert h.factor_device(Ad, m, m, n, Ad, R, precision="fp16") == 0
        assert h.stats()["graph_replay"] == g
        outs.append((from_dev(Ad), R.cpu().numpy()))
    for Q, R in outs[1:]:
        np.testing.assert_array_equal(R, outs[0][1])
        np.testing.assert_array_equal(Q, outs[0][0])


def test_no_graph_for_pageable_buffers_or_profiling(h):
    m, n = 8192, 256
    A = gi.gaussian(m, n, seed=67, dtype="fp16")
    Q = np.empty_like(A, order="F")
    R = np.zeros((n, n), dtype=np.float32, order="F")
    for _ in range(2):
        assert h.factor(A, m, m, n, Q, R, precision="fp16", budget=8 * MiB) == 0
        assert h.stats()["graph_replay"] == 0
    P = Pinned(h, A)
    h.set_option("profile", 1)
    rc, _, _, s = P.factor("fp16", 8 * MiB)
    assert rc == 0 and s["graph_replay"] == 0 and s["kern_launches"][0] > 0
    h.set_option("profile", 0)
    rc, _, _, s = P.factor("fp16", 8 * MiB)
    assert rc == 0 and s["graph_replay"] == 1
    P.free()


@pytest.mark.parametrize("op,tiling,block", [("inner", 0, 2048), ("inner", 1, 128), ("outer", 0, 2048),
                                             ("outer", 1, 256)])
def test_ooc_gemm_graph_replay_equals_eager(h, op, tiling, block):
    """rgsqr_ooc_inner / rgsqr_ooc_outer (Tables 1/2 operations) on page-locked buffers: replays
    equal the eager run bitwise (the outer product updates A2 in place, so each call restarts from
    the same A2)."""
    m, w1, w2 = 16384, 256, 512
    Q = gi.gaussian(m, w1, seed=71, dtype="fp16")
    A = gi.gaussian(m, w2, seed=72, dtype="fp16")
    R = (gi.gaussian(w1, w2, seed=73, dtype="fp32") * 0.05).astype(np.float32)
    pq, pa, pr = h.host_alloc(Q.nbytes), h.host_alloc(A.nbytes), h.host_alloc(R.nbytes)
    vq = np.ctypeslib.as_array((ctypes.c_uint8 * Q.nbytes).from_address(pq))
    va = np.ctypeslib.as_array((ctypes.c_uint8 * A.nbytes).from_address(pa))
    vr = np.ctypeslib.as_array((ctypes.c_uint8 * R.nbytes).from_address(pr))
    vq[:] = Q.reshape(-1, order="F").view(np.uint8)
    outs = []
    for g in (0, 1, 1, 1):
        h.set_option("graph", g)
        va[:] = A.reshape(-1, order="F").view(np.uint8)
        vr[:] = R.reshape(-1, order="F").view(np.uint8)
        if op == "inner":
            h.ooc_inner(pq, m, pa, m, m, w1, w2, pr, w1, precision="fp16", tiling=tiling, block=block,
                        budget=48 * MiB)
        else:
            h.ooc_outer(pq, m, pr, w1, pa, m, m, w1, w2, precision="fp16", tiling=tiling, block=block,
                        budget=48 * MiB)
        assert h.stats()["graph_replay"] == g
        outs.append((va.copy(), vr.copy()))
    for a_, r_ in outs[1:]:
        np.testing.assert_array_equal(a_, outs[0][0])
        np.testing.assert_array_equal(r_, outs[0][1])
    for p_ in (pq, pa, pr):
        h.host_free(p_)

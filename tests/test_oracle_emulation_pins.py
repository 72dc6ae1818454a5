"""Pins for O5 (oracle.rgs_emulated, the precision-emulating recursive CGS) against things
other than itself.  O5 sets GPU acceptance thresholds (tests/test_gpu_*), so it must be
right from BOTH sides: an O5 that forgot a storage rounding would report too small an error
(loosening nothing, but hiding a GPU bug), one that over-rounds would loosen the GPU bounds.

1. Closed form of the backward error (rounding analysis, independent of any emulation):
   with RN-even storage of unit roundoff u, a value with log-uniform mantissa has RMS
   relative rounding error  u * sqrt((4/12) * E[1/f^2]),  f in [1,2) log-uniform,
   E[1/f^2] = (1/ln 2) * (1/2) * (1 - 1/4) = 0.5410,  so  0.4247 u.
   * Storing Q (q_j = u_j/||u_j||, rounded once, R20) perturbs
     A - QR by delta_Q R with ||delta_Q R||_F ~ 0.4247 u ||R||_F = 0.4247 u ||A||_F.
   * Each recursion level (Eq. 2) stores A2' = A2 - Q1 R12 rounded
     (R8); for Gaussian A the A2 blocks of one level hold half of ||A||_F^2,
     so each of the L levels adds (0.4247 u)^2 ||A||_F^2 / 2.
   => backward error  ~=  0.4247 u sqrt(1 + L/2)   (L = levels above the leaves).
   Dropping Q's rounding gives sqrt(L/2 / (1 + L/2)) of it, dropping A2''s 1/sqrt(1+L/2):
   both fail the +-5% bracket at L = 3; dropping both gives fp32 noise.
2. Two-sided brackets against the independent emulation recorded in SURVEY.md:618-626
   (tests/golden/survey_emulation.json), every mode and input class.
3. Structural properties: Q is representable in the storage format (it was stored);
   with a single leaf (L = 0) R is computed in fp32 from exact stored values (DESIGN.md
   R20), so R matches the fp64 R to fp32 level; TF32X3 emulates the RN hi/lo split
   (hi = RN_tf32(x), lo = RN_tf32(x - hi)) that the GPU forms (R25).
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import rgsqr_inputs as gi
from oracle import rgs, rgs_emulated
from oracle.cgs import _mm, _round_tf32_rn, _store

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "survey_emulation.json")))
U = {"fp16": 2.0 ** -11, "bf16": 2.0 ** -8}
RMS_RN = math.sqrt(4.0 / 12.0 * (1.0 / math.log(2.0)) * 0.5 * 0.75)   # 0.4247


def test_rms_rounding_constant():
    # the constant of the closed form, checked by brute force on log-uniform samples
    rng = np.random.default_rng(0)
    x = np.exp2(rng.uniform(0.0, 1.0, 400000)).astype(np.float32) * np.float32(1.37)
    rel = (x.astype(np.float16).astype(np.float64) - x.astype(np.float64)) / x.astype(np.float64)
    assert math.sqrt(np.mean(rel ** 2)) / U["fp16"] == pytest.approx(RMS_RN, rel=0.01)
    assert RMS_RN == pytest.approx(0.4247, abs=1e-4)


@pytest.mark.parametrize("mode", ["fp16", "bf16"])
@pytest.mark.parametrize("m,n,leaf", [(4096, 32, 32), (2048, 128, 32), (4096, 256, 32)])
def test_backward_error_closed_form(mode, m, n, leaf):
    X = gi.to_float64(gi.gaussian(m, n, seed=1, dtype=mode), mode)
    res = rgs_emulated(X, mode, leaf=leaf)
    L = int(round(math.log2(n // leaf)))
    pred = RMS_RN * U[mode] * math.sqrt(1.0 + L / 2.0)
    be = oracle.backward_error(X, res.Q, res.R)
    assert be == pytest.approx(pred, rel=0.05), (be, pred)


@pytest.mark.parametrize("mode", ["fp16", "bf16"])
def test_q_is_stored_in_the_storage_format(mode):
    X = gi.to_float64(gi.gaussian(1024, 128, seed=3, dtype=mode), mode)
    Q = rgs_emulated(X, mode, leaf=32).Q.astype(np.float32)
    np.testing.assert_array_equal(_store(Q, mode), Q)


@pytest.mark.parametrize("mode", ["fp16", "bf16"])
def test_single_leaf_r_is_fp32_accurate(mode):
    # one leaf: no A2' rounding, and the leaf keeps q_j in fp32 until it stores them
    X = gi.to_float64(gi.gaussian(4096, 32, seed=1, dtype=mode), mode)
    assert oracle.r_rel_error(rgs_emulated(X, mode, leaf=32).R, rgs(X, leaf=32).R) < 2e-7


def test_tf32x3_split_is_round_to_nearest():
    rng = np.random.default_rng(5)
    A = rng.standard_normal((64, 48)).astype(np.float32)
    B = rng.standard_normal((48, 40)).astype(np.float32)
    hi = _round_tf32_rn(A)
    lo = _round_tf32_rn(A - hi)
    # both parts are tf32 numbers (low 13 mantissa bits clear) and hi is the nearest one
    assert np.all(hi.view(np.uint32) & 0x1FFF == 0) and np.all(lo.view(np.uint32) & 0x1FFF == 0)
    assert np.all(np.abs(A - hi) <= np.abs(A) * 2.0 ** -11)
    assert np.all(np.abs(A - hi - lo) <= np.abs(A) * 2.0 ** -22)
    exact = A.astype(np.float64) @ B.astype(np.float64)
    err3 = np.abs(_mm(A, B, "tf32x3") - exact).max() / np.abs(exact).max()
    err1 = np.abs(_mm(A, B, "tf32") - exact).max() / np.abs(exact).max()
    assert err3 < 2e-6 < 1e-4 < err1


CASES = [("gaussian", None), ("kappa_10", 10.0), ("kappa_1000", 1e3)]


@pytest.mark.parametrize("mode", ["fp16", "bf16", "tf32", "tf32x3"])
@pytest.mark.parametrize("case,kappa", CASES)
def test_two_sided_bracket_vs_survey_emulation(mode, case, kappa):
    m, n, leaf = GOLD["m"], GOLD["n"], GOLD["leaf"]
    st = mode if mode in ("fp16", "bf16") else "fp32"
    if kappa is None:
        X = gi.to_float64(gi.gaussian(m, n, seed=1, dtype=st), st)
    else:
        A, _ = gi.usv(m, n, kappa=kappa, seed=1)
        X = gi.to_float64(gi.to_storage(A.astype(np.float32), st), st)
    res = rgs_emulated(X, mode, leaf=leaf)
    ref = rgs(X, leaf=leaf)
    got = [oracle.backward_error(X, res.Q, res.R), oracle.r_rel_error(res.R, ref.R), oracle.orthogonality(res.Q)]
    for name, g, s in zip(("backward", "R", "orth"), got, GOLD[case][mode]):
        assert s / 1.6 <= g <= s * 1.6, f"{case} {mode} {name}: {g:.3e} vs survey {s:.3e}"

"""Pins for oracle/model.py against numbers printed in the paper (tests/golden/)."""
import json
import os

import pytest

from oracle import model

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_numbers.json")))


def test_recursion_shapes_paper_example():
    g = GOLD["inner_product_shapes_131072sq_b8192"]
    shapes = model.recursion_inner_products(g["m"], g["n"], g["b"])
    assert sorted({tuple(s) for s in shapes}) == sorted(tuple(s) for s in g["distinct_shapes"])
    # one product of width 65536, two of 32768, four of 16384, eight of 8192
    counts = {}
    for w1, _, _ in shapes:
        counts[w1] = counts.get(w1, 0) + 1
    assert counts == {65536: 1, 32768: 2, 16384: 4, 8192: 8}


@pytest.mark.parametrize("m,n,b", [(131072, 131072, 8192), (65536, 8192, 64), (4096, 256, 32)])
def test_flops_sum_to_2mn2(m, n, b):
    assert model.recursion_flops(m, n, b) == model.flops(m, n)


def test_table1_flop_convention():
    g = GOLD["table1_inner_recursive"]
    blk = 2.0 * g["gemm_m"] * g["block"] * g["gemm_n"] / (g["block_gemm_ms"] / 1e3) / 1e12
    tot_async = 2.0 * g["gemm_m"] * g["gemm_k"] * g["gemm_n"] / (g["async_ms"] / 1e3) / 1e12
    tot_sync = 2.0 * g["gemm_m"] * g["gemm_k"] * g["gemm_n"] / (g["sync_ms"] / 1e3) / 1e12
    assert round(blk, 1) == pytest.approx(g["block_gemm_tflops"], abs=0.1)
    assert round(tot_async, 1) == g["async_tflops"]
    assert tot_sync == pytest.approx(g["sync_tflops"], abs=0.1)   # paper prints 62.0 for 61.92


def test_table2_ideal_time():
    g = GOLD["table2_outer_recursive"]
    nblk = g["gemm_m"] // g["block"]
    assert g["block_gemm_ms"] * nblk + g["h2d_ms"] + g["d2h_ms"] == g["ideal_ms"]
    tot = 2.0 * g["gemm_m"] * g["gemm_k"] * g["gemm_n"] / (g["async_ms"] / 1e3) / 1e12
    assert tot == pytest.approx(g["async_tflops"], abs=0.1)     # paper truncates 97.76


def test_overlap_condition():
    g = GOLD["overlap_condition_v100"]
    assert model.inner_overlap_condition(g["rg"], g["rm"], 4) == g["m_min"]


@pytest.mark.parametrize("m,n,b", [(1000, 64, 8), (4096, 256, 32), (65536, 8192, 1024), (7, 12, 3)])
def test_blocked_closed_form_equals_iteration_sum(m, n, b):
    k = n // b
    h = d = 0
    for i in range(1, k + 1):
        hi, di = model.blocked_iteration_words(m, n, b, i)
        h += hi
        d += di
    H, D = model.blocked_total_words(m, n, b)
    assert h == H and d == D


@pytest.mark.parametrize("m,n,b", [(1000, 64, 8), (4096, 256, 32), (65536, 8192, 1024), (3, 32, 1)])
def test_recursive_closed_form_equals_count(m, n, b):
    assert model.recursive_noreuse_words_count(m, n, b) == model.recursive_noreuse_words_closed(m, n, b)


def test_recursive_k1_equals_blocked_k1():
    # one panel: both strategies read A once and write Q + R once
    assert model.recursive_noreuse_words_count(500, 16, 16) == (500 * 16, 500 * 16 + 256)
    h, d = model.blocked_total_words(500, 16, 16)
    assert d == 500 * 16 + 256


def test_recursive_moves_less_than_blocked():
    # PAPER.md:155 / Table 3 claim, for k >= 4
    for m, n, b in [(131072, 131072, 16384), (131072, 131072, 8192), (65536, 65536, 8192)]:
        rh, rd = model.recursive_noreuse_words_closed(m, n, b)
        bh, bd = model.blocked_total_words(m, n, b)
        assert rh < bh and rd < bd


def _r12_words(m, n, b):
    """Sum of w1*w2 over the recursion's inner products (the R12 words the paper's outer
    product re-reads: 'outer reads Q1 + R12 + A2')."""
    return sum(w1 * w2 for w1, _, w2 in model.recursion_inner_products(m, n, b))


@pytest.mark.parametrize("m,n,b", [(1000, 64, 8), (4096, 256, 32), (65536, 8192, 64), (7, 12, 3), (100, 96, 32)])
def test_recursive_split_words_identity(m, n, b):
    """The executor-shaped split (GPU byte-counter target, tests/test_gpu_factor_host.py)
    differs from the paper-accounting count (reading R11 of PAPER.md:147-153, itself pinned
    to its closed form above) by exactly the R12 re-reads of the outer product, which the
    executor does not do because R12 stays resident."""
    sp = model.recursive_noreuse_split_words(m, n, b)
    h, d = model.recursive_noreuse_words_count(m, n, b)
    assert sp["h2d_matrix"] + _r12_words(m, n, b) == h
    assert sp["d2h_matrix"] + sp["d2h_r"] == d


@pytest.mark.parametrize("m,n,b", [(1000, 64, 8), (4096, 256, 32), (65536, 8192, 1024), (131072, 131072, 8192)])
def test_blocked_split_words_identity(m, n, b):
    """blocked split + the R12 re-reads sum_i b(n - ib) + the last panel's 2mb (PAPER.md:139
    counts mb + mb + mb for it although there is no trailing matrix) == PAPER.md:141 exactly;
    its D2H == PAPER.md:145 exactly."""
    k = n // b
    sp = model.blocked_noreuse_split_words(m, n, b)
    H, D = model.blocked_total_words(m, n, b)
    assert sp["h2d_matrix"] + sum(b * (n - i * b) for i in range(1, k + 1)) + 2 * m * b == H
    assert sp["d2h_matrix"] + sp["d2h_r"] == D

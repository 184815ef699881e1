"""Pins for oracle/sums.py against closed forms, invariants, exact arithmetic and a library routine."""
import math

import numpy as np
import pytest
import torch

from oracle import sums
from synth import gen

SHAPES = [(1, 1), (1, 7), (7, 1), (3, 5), (31, 33), (33, 31), (64, 100), (100, 64)]


@pytest.mark.parametrize("R,C", SHAPES)
def test_ones_closed_form(R, C):
    m = np.ones((R, C), dtype=np.float32)
    assert sums.sum_rows(m).tolist() == [float(C)] * R
    assert sums.sum_cols(m).tolist() == [float(R)] * C
    assert sums.sum_rows_literal(m) == [float(C)] * R
    assert sums.sum_cols_literal(m) == [float(R)] * C
    mi = np.ones((R, C), dtype=np.int32)
    assert sums.sum_rows(mi).tolist() == [C] * R
    assert sums.sum_cols(mi).tolist() == [R] * C


@pytest.mark.parametrize("R,C", SHAPES + [(1000, 777)])
def test_arange_closed_form_int64(R, C):
    # m[r,c] = r*C + c: rowsum = r*C^2 + C(C-1)/2, colsum = C*R(R-1)/2 + R*c
    m = gen.arange_matrix((R, C), torch.int64).numpy()
    rows = sums.sum_rows(m).tolist()
    cols = sums.sum_cols(m).tolist()
    assert rows == [r * C * C + C * (C - 1) // 2 for r in range(R)]
    assert cols == [C * R * (R - 1) // 2 + R * c for c in range(C)]
    if R * C <= 4096:
        assert sums.sum_rows_literal(m) == rows
        assert sums.sum_cols_literal(m) == cols


def test_arange_int32_wraps():
    # values r*C + c wrapped to int32 (offset pushes past 2^31); sums wrap mod 2^32
    R, C = 300, 257
    off = (1 << 31) - 5000
    m = gen.arange_matrix((R, C), torch.int32, offset=off).numpy()
    rows = sums.sum_rows(m).tolist()
    cols = sums.sum_cols(m).tolist()
    for r in range(0, R, 37):
        exact = sum(off + r * C + c for c in range(C))
        assert rows[r] == sums.wrap(exact, 32)
    for c in range(0, C, 41):
        exact = sum(off + r * C + c for r in range(R))
        assert cols[c] == sums.wrap(exact, 32)
    assert sums.sum_rows_literal(m[:5]) == rows[:5]


def test_int64_wide_wraps_mod_2_64():
    m = gen.int64_wide(9, (17, 23)).numpy()
    for r in range(17):
        assert sums.sum_rows(m)[r] == sums.wrap(sum(int(v) for v in m[r]), 64)
    for c in range(23):
        assert sums.sum_cols(m)[c] == sums.wrap(sum(int(v) for v in m[:, c]), 64)


@pytest.mark.parametrize("R,C", [(31, 33), (257, 100), (64, 1000)])
def test_total_invariance(R, C):
    mi = gen.int_uniform(2, (R, C), -1000, 1000).numpy()
    assert int(sums.sum_rows(mi).astype(np.int64).sum()) == int(sums.sum_cols(mi).astype(np.int64).sum())
    mf = gen.uniform_f32(1, (R, C)).numpy()
    assert math.isclose(math.fsum(sums.sum_rows(mf)), math.fsum(sums.sum_cols(mf)), rel_tol=1e-13)
    # arange: Σ = RC(RC−1)/2
    ma = gen.arange_matrix((R, C), torch.int64).numpy()
    assert int(sums.sum_rows(ma).sum()) == R * C * (R * C - 1) // 2


def test_exact_summable_fp32_is_exact():
    # k * 2^-8 with k < 256: every partial sum of <= 65,536 terms is exact in fp32 and fp64
    m = gen.exact_f32(11, (300, 700)).numpy()
    rows = sums.sum_rows(m)
    cols = sums.sum_cols(m)
    ref_rows = [sum(int(round(v * 256)) for v in m[r]) / 256.0 for r in range(300)]
    ref_cols = [sum(int(round(v * 256)) for v in m[:, c]) / 256.0 for c in range(700)]
    assert rows.tolist() == ref_rows
    assert cols.tolist() == ref_cols


@pytest.mark.parametrize("R,C", [(1, 1), (2, 3), (3, 2), (31, 32), (33, 64), (100, 3)])
def test_literal_vs_bruteforce_and_library(R, C):
    m = gen.uniform_f32(3, (R, C)).numpy()
    lit_r, lit_c = sums.sum_rows_literal(m), sums.sum_cols_literal(m)
    t = torch.from_numpy(m).double()
    lib_r, lib_c = t.sum(1).tolist(), t.sum(0).tolist()        # library routine (torch CPU fp64)
    vec_r, vec_c = sums.sum_rows(m).tolist(), sums.sum_cols(m).tolist()
    for a, b, c in zip(lit_r, lib_r, vec_r):
        assert math.isclose(a, b, rel_tol=1e-14) and math.isclose(a, c, rel_tol=1e-14)
    for a, b, c in zip(lit_c, lib_c, vec_c):
        assert math.isclose(a, b, rel_tol=1e-14) and math.isclose(a, c, rel_tol=1e-14)


def test_transpose_relation():
    # sumCols(m) == sumRows(m^T): catches a transposed operand in either function
    m = gen.int_uniform(4, (37, 19), -50, 50).numpy()
    assert sums.sum_cols(m).tolist() == sums.sum_rows(np.ascontiguousarray(m.T)).tolist()


@pytest.mark.parametrize("n,k", [(10, 3), (10, 4), (10, 6), (7, 7), (65536, 10), (1, 1)])
def test_split_chunks(n, k):
    ch = sums.split_chunks(n, k)
    L = -(-n // k)
    assert ch[0][0] == 0 and ch[-1][1] == n
    assert all(e - s == L for s, e in ch[:-1]) and 0 < ch[-1][1] - ch[-1][0] <= L
    assert all(ch[i][1] == ch[i + 1][0] for i in range(len(ch) - 1))


@pytest.mark.parametrize("pattern", ["rows", "cols"])
def test_split_partials_sum_to_total(pattern):
    m = gen.int_uniform(5, (50, 70), -100, 100).numpy()
    p = sums.split_partials(m, pattern, 4).view(np.int64)
    total = sums.sum_rows(m) if pattern == "rows" else sums.sum_cols(m)
    assert p.sum(axis=0).tolist() == total.tolist()
    # white box: partial 1 of rows covers columns [18, 36)
    if pattern == "rows":
        assert p[1].tolist() == m[:, 18:36].astype(np.int64).sum(axis=1).tolist()


def test_weighted_closed_forms():
    R, C = 40, 30
    m = np.ones((R, C), dtype=np.float32)
    v = np.arange(C, dtype=np.float32)
    assert sums.sum_weighted_rows(m, v).tolist() == [C * (C - 1) / 2] * R
    vr = np.arange(R, dtype=np.float32)
    assert sums.sum_weighted_cols(m, vr).tolist() == [R * (R - 1) / 2] * C
    # v = 1 reduces to the plain sums
    mf = gen.uniform_f32(7, (R, C)).numpy()
    assert np.allclose(sums.sum_weighted_rows(mf, np.ones(C, np.float32)), sums.sum_rows(mf), rtol=1e-15)
    assert np.allclose(sums.sum_weighted_cols(mf, np.ones(R, np.float32)), sums.sum_cols(mf), rtol=1e-15)
    mi = gen.int_uniform(8, (R, C), -9, 9).numpy()
    vi = gen.int_uniform(9, (C,), -9, 9).numpy()
    assert sums.sum_weighted_rows(mi, vi).tolist() == sums.sum_weighted_rows_literal(mi, vi)
    vri = gen.int_uniform(10, (R,), -9, 9).numpy()
    assert sums.sum_weighted_cols(mi, vri).tolist() == sums.sum_weighted_cols_literal(mi, vri)


@pytest.mark.parametrize("R,C", [(1, 1), (3, 5), (33, 31), (100, 64)])
def test_rows_cols_closed_forms(R, C):
    # sumRowsCols (Naive Bayes counts, §VI-E) = [sumRows | sumCols]: ones give C per row and
    # R per column; arange m[r,c] = r*C + c gives r*C^2 + C(C-1)/2 and C*R(R-1)/2 + R*c; both halves
    # total RC(RC-1)/2; the literal nested loops agree
    ones = np.ones((R, C), dtype=np.int32)
    assert sums.sum_rows_cols(ones).tolist() == [C] * R + [R] * C
    a = np.arange(R * C, dtype=np.int64).reshape(R, C)
    want = [r * C * C + C * (C - 1) // 2 for r in range(R)] + [C * R * (R - 1) // 2 + R * c for c in range(C)]
    got = sums.sum_rows_cols(a)
    assert got.tolist() == want
    assert int(got[:R].sum()) == int(got[R:].sum()) == R * C * (R * C - 1) // 2
    assert sums.sum_rows_cols_literal(a) == want

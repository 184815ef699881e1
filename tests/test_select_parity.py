"""C++ selector (libnpp.so npp_select, no GPU needed) == oracle selector, record by record."""
import itertools

import pytest

from oracle import select as S

npp = pytest.importorskip("paper_conf_micro_leebsro14_b200.npp")

TINY = dict(sm_count=2, max_threads_per_sm=1024, max_threads_per_block=256, max_block_dim=(256, 256, 64),
            warp_size=32, max_blocks_per_sm=8, regs_per_sm=32768, regs_per_block=32768, regs_per_thread=40,
            smem_per_block=16384)
B200_64 = dict(S.B200, regs_per_thread=64)
PROFILES = {"b200": S.B200, "b200_64regs": B200_64, "k20c": S.K20C, "tiny": TINY}

SIZES = [1, 2, 3, 31, 32, 33, 100, 1000, 1024, 4096, 65536, 1 << 20]
SUM_STRATS = ["AUTO", "LITERAL", "1D", "TB_T", "WARP"]


def _cmp(pattern, shape, dtype, lim, strat):
    try:
        want = S.select(pattern, shape, dtype, lim, strat)
    except S.NoFeasibleMapping:
        with pytest.raises(npp.NppError) as e:
            npp.select(pattern, shape, dtype, lim, strat)
        assert e.value.status == npp.ERR_NO_FEASIBLE
        return
    except S.Unsupported:
        with pytest.raises(npp.NppError) as e:
            npp.select(pattern, shape, dtype, lim, strat)
        assert e.value.status == npp.ERR_UNSUPPORTED
        return
    got = npp.select(pattern, shape, dtype, lim, strat)
    assert got == want, (pattern, shape, dtype, strat)


@pytest.mark.parametrize("profile", list(PROFILES))
@pytest.mark.parametrize("pattern", ["SUM_ROWS", "SUM_COLS", "SUM_WEIGHTED_ROWS", "SUM_WEIGHTED_COLS",
                                     "SUM_ROWS_COLS"])
def test_sums_exhaustive(profile, pattern):
    lim = PROFILES[profile]
    for R, C in itertools.product(SIZES, SIZES):
        if R * C > (1 << 34):
            continue
        for dtype in ("f32", "i32", "i64", "f64"):
            for strat in SUM_STRATS:
                _cmp(pattern, (R, C), dtype, lim, strat)


@pytest.mark.parametrize("profile", list(PROFILES))
def test_three_level_literal(profile):
    lim = PROFILES[profile]
    for shape in [(1 << 22, 64, 32), (1000, 3, 5), (17, 256, 1), (64, 1, 64), (4096 * 4096, 64, 32),
                  (4099, 128, 96), (20000, 64, 256), (10, 128, 256)]:
        for strat in ("LITERAL", "AUTO"):
            _cmp("KMEANS_ASSIGN", shape, "f32", lim, strat)
    for shape in [(4096, 4096, 256), (1, 1 << 24, 256), (3, 7, 5), (512, 4096, 256), (7, 33, 100),
                  (2, 5, 512), (64, 32, 4)]:
        for strat in ("LITERAL", "AUTO"):
            _cmp("LOGREG_GRAD", shape, "f32", lim, strat)
    for strat in ("1D", "TB_T", "WARP"):
        _cmp("KMEANS_ASSIGN", (1000, 64, 32), "f32", lim, strat)


@pytest.mark.parametrize("profile", list(PROFILES))
def test_kmeans_update_parity(profile):
    lim = PROFILES[profile]
    for shape in [(1 << 22, 64, 32), (1000, 3, 5), (17, 64, 1), (64, 4, 256), (4099, 60, 34), (128, 64, 33),
                  (1, 8, 8), (300, 128, 4), (5000, 16, 300)]:
        for strat in SUM_STRATS:
            _cmp("KMEANS_UPDATE", shape, "f32", lim, strat)


@pytest.mark.parametrize("profile", list(PROFILES))
def test_pagerank_parity(profile):
    lim = PROFILES[profile]
    for shape in [(1 << 22, 70000000), (1000, 0), (1, 5), (7, 7), (5000, 80000), (100, 100000), (33, 1 << 20),
                  (1 << 20, 1 << 20), (1000, 16000, 4000), (1, 3, 1 << 22)]:
        for strat in SUM_STRATS:
            _cmp("PAGERANK", shape, "f32", lim, strat)


def test_unknown_sizes_literal():
    for shape in [(-1, 1024), (1024, -1), (-1, -1)]:
        for pattern in ("SUM_ROWS", "SUM_COLS"):
            _cmp(pattern, shape, "f32", S.B200, "LITERAL")


def test_invalid_arguments():
    with pytest.raises(npp.NppError) as e:
        npp.select("SUM_ROWS", (0, 4), "f32", S.B200, "AUTO")
    assert e.value.status == npp.ERR_INVALID_ARG
    with pytest.raises(npp.NppError) as e:
        npp.select("SUM_ROWS", (4, 4, 4), "f32", S.B200, "AUTO")
    assert e.value.status == npp.ERR_INVALID_ARG
    with pytest.raises(npp.NppError) as e:
        npp.select("SUM_ROWS", (4, 4), "f32", dict(S.B200, sm_count=0), "AUTO")
    assert e.value.status == npp.ERR_INVALID_ARG
    with pytest.raises(npp.NppError) as e:
        npp.select("KMEANS_ASSIGN", (4, 4, 4), "i32", S.B200, "LITERAL")
    assert e.value.status == npp.ERR_UNSUPPORTED


@pytest.mark.parametrize("profile", ["b200", "k20c", "tiny"])
def test_enumerate_parity(profile):
    # npp_enumerate (Fig 17 sweep space) == oracle enumeration, record by record and in order
    lim = PROFILES[profile]
    for pattern in ("SUM_ROWS", "SUM_COLS", "SUM_WEIGHTED_COLS", "SUM_ROWS_COLS"):
        for shape in [(65536, 1024), (1024, 65536), (50, 20000), (3, 5)]:
            for dtype in ("f32", "i64"):
                want = S.enumerate_mappings(pattern, shape, dtype, lim)
                got = npp.enumerate_mappings(pattern, shape, dtype, lim)
                assert got == want, (pattern, shape, dtype)
    for pattern, shape in [("KMEANS_ASSIGN", (1000, 8, 4)), ("LOGREG_GRAD", (4, 64, 8))]:
        assert npp.enumerate_mappings(pattern, shape, "f32", lim) == S.enumerate_mappings(pattern, shape, "f32", lim)


def test_enumerate_contains_the_selection():
    # the LITERAL selection is the S5-best member of the enumerated space (same record)
    for pattern, shape in [("SUM_ROWS", (8192, 8192)), ("SUM_COLS", (65536, 1024)), ("SUM_COLS", (1024, 65536))]:
        space = npp.enumerate_mappings(pattern, shape, "f32", S.B200)
        lit = npp.select(pattern, shape, "f32", S.B200, "LITERAL")
        assert lit in space
        assert lit["score"] == max(r["score"] for r in space)
    assert npp.enumerate_mappings("SUM_ROWS", (3, 5), "f32", S.B200)  # never empty for feasible nests

"""Pins of the runtime rule R2 (S8; the paper's "dynamic decision" of block sizes and
span/split factors) by properties the kernels rely on, over a grid of shapes x dtypes x
device profiles. R2 is a B200 design choice the paper does not print, so it is pinned by what any
correct schedule must satisfy, not by values:

  * the static ranges and the claim-pool units cover every tile of To x Ti exactly once;
  * every outer tile's contributions add up to its Ti tiles (the ticket target of the fused Split
    combine, P:L542-550 / L880-883); for LOGREG_GRAD the ticket target the kernel computes equals the
    number of distinct blocks that cover the batch;
  * the whole-tile rules (RX one-row tiles, MX-narrow strips) never cut an outer tile;
  * tiles fill one 32 KB ring slot and cover the matrix; blocks get balanced work;
  * a vector width V divides every chunk of the level on x, and Split chunks leave no block empty;
  * workspace_bytes covers every byte the kernel addresses (pool counter, tickets, accumulators).

A plausible slip in R2 (an off-by-one in a range bound, a Ts that is not a multiple of the unit, a
ticket formula counting tiles instead of blocks, a workspace section sized for the wrong level)
fails one of these.
"""
import itertools

import pytest

from oracle import select as S
from schedule import (ESZ, cdiv, contiguous_ranges, pool_units, rc_regions, staged_geometry,
                            static_ranges)

TINY = dict(sm_count=2, max_threads_per_sm=1024, max_threads_per_block=256, max_block_dim=(256, 256, 64),
            warp_size=32, max_blocks_per_sm=8, regs_per_sm=32768, regs_per_block=32768, regs_per_thread=40,
            smem_per_block=16384)
PROFILES = {"b200": S.B200, "k20c": S.K20C, "tiny": TINY}
SIZES = [1, 3, 31, 32, 33, 100, 1000, 1024, 4097, 8192, 65536, 1 << 20]


def _select(pattern, shape, dtype, lim):
    try:
        return S.select(pattern, shape, dtype, lim, "AUTO")
    except (S.Unsupported, S.NoFeasibleMapping):
        return None


def _check_staged_sum(pattern, shape, dtype, lim, rec):
    R, C = shape
    esz = ESZ[dtype]
    rows = pattern in ("SUM_ROWS", "SUM_WEIGHTED_ROWS")
    To, Ti, BR, W, align = staged_geometry(pattern, shape, dtype, rec)
    T, G, U, Ts = To * Ti, rec["grid"], rec["claim_tiles"], rec["static_tiles"]
    # tiles: one 32 KB ring slot each, covering the matrix with at most one partial tile per level
    assert BR * W * esz == 32768, (BR, W)
    outer_extent, inner_extent = (R, C) if rows else (C, R)
    outer_tile, inner_tile = (BR, W) if rows else (W, BR)
    assert cdiv(outer_extent, outer_tile) == To and cdiv(inner_extent, inner_tile) == Ti
    # grid and pool
    assert 1 <= G <= min(lim["sm_count"], T)
    assert 1 <= U and 0 <= Ts <= T
    assert T - Ts <= T // 8 + U, "the pool holds about 1/8 of the tiles"
    ranges = static_ranges(G, Ts, Ti, align)
    # static ranges partition [0, Ts) in block order
    assert ranges[0][0] == 0 and ranges[-1][1] == Ts
    assert all(a[1] == b[0] for a, b in zip(ranges, ranges[1:]))
    assert all(s0 <= s1 for s0, s1 in ranges)
    sizes = [s1 - s0 for s0, s1 in ranges]
    assert max(sizes) - min(sizes) <= (Ti if align else 1), "balanced static split"
    units = pool_units(T, Ts, U, Ti, G)
    assert units == S.pool_claims(T, Ts, U, Ti, G)
    # the blocks end within one tile of each other when outer tiles may be cut: the final claims are
    # single tiles, at least one per block (or every pool tile)
    if U < Ti:
        assert all(e - s0 == 1 for s0, e in units[-min(G, T - Ts):])
    # exact cover of [0, T)
    seen = [0] * T
    for s0, s1 in ranges + units:
        for t in range(s0, s1):
            seen[t] += 1
    assert all(v == 1 for v in seen)
    # whole-tile rules never cut an outer tile: every segment is a union of whole outer tiles
    if align:
        assert U == Ti and Ts % Ti == 0
        for s0, s1 in ranges + units:
            assert s0 % Ti == 0 and (s1 % Ti == 0 or s1 == T)
    # per outer tile: the contributions (tile counts the combiner adds to the ticket) total Ti
    contrib = [0] * To
    for s0, s1 in ranges + units:
        for o in range(s0 // Ti, cdiv(s1, Ti)):
            contrib[o] += max(0, min(s1, (o + 1) * Ti) - max(s0, o * Ti))
    assert contrib == [Ti] * To
    # workspace: pool counters (256 B), tickets [To] u32, accumulators [O] (fp64 / u32 / u64)
    O = R if rows else C
    ab = 4 if dtype == "i32" else 8
    need = 256 + 256 * cdiv(4 * To, 256) + O * ab
    assert rec["workspace_bytes"] >= need
    # the x level streams 16-byte vectors (RX) or one column per thread (MX)
    assert rec["vec"] == (16 // esz if rows else 1)


def _check_unstaged_sum(pattern, shape, dtype, lim, rec):
    R, C = shape
    rows = pattern in ("SUM_ROWS", "SUM_WEIGHTED_ROWS")
    O, I = (R, C) if rows else (C, R)
    lo, li = rec["levels"]
    x_level = 0 if lo["dim"] == S.X else 1
    V = rec["vec"]
    if V > 1:  # vectors only along the stride-1 x level and with a 16-B row pitch
        assert x_level == (1 if rows else 0) and C % V == 0 and V == 16 // ESZ[dtype]
    lx = rec["levels"][x_level]
    assert lx["chunk"] % V == 0 or lx["chunk"] == (I if x_level == 1 else O)
    # every block of a level has work: chunk * grid covers the level, (grid - 1) * chunk does not
    for lv, n in ((lo, O), (li, I)):
        assert lv["grid"] * lv["chunk"] >= n > (lv["grid"] - 1) * lv["chunk"]
    if x_level == 1:  # RX: shuffle reduction over min(b_x, 32) lanes
        bx = li["block"]
        assert (bx <= 32 and bx & (bx - 1) == 0) or bx % 32 == 0
    assert lo["block"] * li["block"] <= lim["max_threads_per_block"]
    if li["grid"] >= 2:  # Split: partials [gi x O] + tickets [go]
        ab = 4 if dtype == "i32" else 8
        need = 256 * cdiv(li["grid"] * O * ab, 256) + 4 * lo["grid"]
        assert rec["workspace_bytes"] >= need
        assert li["span"] == S.SPLIT and li["factor"] == li["grid"]


@pytest.mark.parametrize("profile", list(PROFILES))
@pytest.mark.parametrize("pattern", ["SUM_ROWS", "SUM_COLS", "SUM_WEIGHTED_ROWS", "SUM_WEIGHTED_COLS"])
def test_sum_schedules(profile, pattern):
    lim = PROFILES[profile]
    n_staged = 0
    for R, C in itertools.product(SIZES, SIZES):
        if R * C > (1 << 30):
            continue
        for dtype in ("f32", "i32", "i64", "f64"):
            rec = _select(pattern, (R, C), dtype, lim)
            if rec is None:
                continue
            if rec["staged"]:
                n_staged += 1
                _check_staged_sum(pattern, (R, C), dtype, lim, rec)
            else:
                assert rec["static_tiles"] == 0
                _check_unstaged_sum(pattern, (R, C), dtype, lim, rec)
    assert n_staged > 50


def test_paper_shape_schedules_use_every_rule():
    # the paper shapes exercise the narrow, wide, one-row and MX-narrow tile rules (S8)
    kinds = set()
    for pattern in ("SUM_ROWS", "SUM_COLS"):
        for shape in [(65536, 1024), (8192, 8192), (1024, 65536), (1 << 20, 4096)]:
            rec = S.select(pattern, shape, "f32", S.B200, "AUTO")
            To, Ti, BR, W, align = staged_geometry(pattern, shape, "f32", rec)
            kinds.add((pattern, BR, align))
            _check_staged_sum(pattern, shape, "f32", S.B200, rec)
    assert ("SUM_ROWS", 1, True) in kinds and ("SUM_COLS", 128, True) in kinds
    assert ("SUM_ROWS", 8, False) in kinds and ("SUM_COLS", 32, False) in kinds


@pytest.mark.parametrize("profile", list(PROFILES))
def test_logreg_schedules(profile):
    lim = PROFILES[profile]
    for B, Rb, C in [(4096, 4096, 256), (1, 1 << 20, 256), (3, 7, 8), (7, 33, 100), (512, 4096, 256),
                     (64, 32, 4), (1000, 100, 12), (5, 1000, 256), (150, 64, 64)]:
        rec = _select("LOGREG_GRAD", (B, Rb, C), "f32", lim)
        if rec is None:
            assert lim is not S.B200 or C % 4 or C > 256
            continue
        Ti = cdiv(Rb, 32)
        T, P, G = B * Ti, rec["claim_tiles"], rec["grid"]
        assert G <= lim["sm_count"] and G * P >= T > (G - 1) * P
        ranges = contiguous_ranges(T, P, G)
        assert ranges[-1][1] == T and all(s1 > s0 for s0, s1 in ranges)
        for b in range(B):
            f0, f1 = b * Ti, (b + 1) * Ti
            distinct = {t // P for t in range(f0, f1)}
            # the ticket target the LR kernel computes for a cut batch (kern_logreg.cu)
            assert (f1 - 1) // P - f0 // P + 1 == len(distinct)
        assert rec["workspace_bytes"] >= 256 * cdiv(4 * B, 256) + 8 * B * C


@pytest.mark.parametrize("profile", list(PROFILES))
def test_kmeans_schedules(profile):
    lim = PROFILES[profile]
    for N, D, K in [(1 << 22, 64, 32), (1000, 4, 1), (257, 64, 256), (4099, 128, 96), (20000, 64, 256),
                    (10, 128, 128), (1, 8, 3), (300000, 68, 33)]:
        rec = _select("KMEANS_ASSIGN", (N, D, K), "f32", lim)
        if rec is None:  # unsupported shapes, or a profile that cannot hold the block (threads, regs, smem)
            assert lim is not S.B200 or D % 4 or D > 128 or K > 256 or 32 * cdiv(K, 32) * D > 16384
            assert (D % 4 or D > 128 or K > 256 or 32 * cdiv(K, 32) * D > 16384 or lim["max_threads_per_block"] < 512
                    or lim["smem_per_block"] < S.km_smem_bytes(K, D, 2))
            continue
        TP = 256 if D <= 64 else 128
        T, P, G = cdiv(N, TP), rec["claim_tiles"], rec["grid"]
        assert G <= lim["sm_count"] and G * P >= T > (G - 1) * P
        assert 32 * cdiv(K, 32) * D <= 16384  # the centroid pairs fit the 64 KB constant bank
        # warp sets: three only when every set reads the same (single) 32-centroid chunk; a block of
        # S sets x 256 threads covers S tiles at once (TP/64 points per thread)
        S_ = 3 if K <= 32 and lim["max_threads_per_block"] >= 768 else 2
        l0 = rec["levels"][0]
        assert l0["block"] * rec["levels"][1]["block"] == 256 * S_
        assert l0["chunk"] == S_ * TP == l0["block"] * l0["factor"]
        assert 256 * S_ * 80 <= lim["regs_per_block"]  # the 80-register cap keeps the block resident
        assert S.km_smem_bytes(K, D, S_) <= lim["smem_per_block"]


@pytest.mark.parametrize("profile", list(PROFILES))
def test_kmeans_update_schedules(profile):
    lim = PROFILES[profile]
    for N, D, K in [(1 << 22, 64, 32), (1000, 4, 1), (129, 64, 32), (5000, 16, 128), (1, 8, 8), (77777, 60, 34)]:
        rec = _select("KMEANS_UPDATE", (N, D, K), "f32", lim)
        assert rec is not None
        T, P, G = cdiv(N, 96), rec["claim_tiles"], rec["grid"]
        assert G <= lim["sm_count"] and G * P >= T > (G - 1) * P
        assert rec["workspace_bytes"] >= 256 + 8 * K * (D + 1)
        assert [lv["block"] for lv in rec["levels"]] == [12, 32]  # 12 consumer warps, 8 points each per tile
        assert K * D <= 2048  # twelve warp-private fp32 [K x D] copies in 96 KB of shared memory


@pytest.mark.parametrize("profile", list(PROFILES))
def test_rowscols_schedules(profile):
    lim = PROFILES[profile]
    for R, C in itertools.product([1, 31, 33, 1000, 8192, 65536], [1, 4, 257, 1024, 8192, 65536]):
        for dtype in ("f32", "i32", "i64", "f64"):
            rec = _select("SUM_ROWS_COLS", (R, C), dtype, lim)
            if rec is None:
                continue
            BC = 1024 // ESZ[dtype]
            Tr, Tc = cdiv(R, 32), cdiv(C, BC)
            gr, gc, nreg, G, ranges = rc_regions(rec)
            cr = cdiv(rec["levels"][0]["chunk"], 32) if gr > 1 else Tr
            cc = cdiv(rec["levels"][1]["chunk"], BC) if gc > 1 else Tc
            assert gr * cr >= Tr > (gr - 1) * cr and gc * cc >= Tc > (gc - 1) * cc
            assert cc <= 32, "a region's column accumulators fit shared memory"
            assert G <= lim["sm_count"] and G <= nreg
            assert ranges[0][0] == 0 and ranges[-1][1] == nreg
            assert all(s1 > s0 for s0, s1 in ranges) and all(a[1] == b[0] for a, b in zip(ranges, ranges[1:]))
            assert rec["claim_tiles"] == cr * cc
            ab = 4 if dtype == "i32" else 8
            assert rec["workspace_bytes"] >= 4 * gr + 4 * gc + (R + C) * ab


@pytest.mark.parametrize("profile", list(PROFILES))
def test_pagerank_schedules(profile):
    lim = PROFILES[profile]
    for shape in [(1 << 22, 70000000), (1000, 0), (1, 5), (7, 7), (5000, 80000), (100, 100000),
                  (1000, 16000, 4000)]:
        rec = _select("PAGERANK", shape, "f32", lim)
        N = shape[0]
        V = rec["levels"][1]["block"]
        chunk = rec["claim_tiles"]
        m = rec["levels"][1]["chunk"]  # mean in-degree ceil(E/N)
        if m >= 8:  # segmented: 32 lanes split a chunk of 31 rows' edges; lane i of a claim holds row i
            assert rec["levels"][1]["span"] == S.SPLIT and V == 32 and rec["levels"][0]["block"] == 8
            assert chunk == 31 and chunk < 32 and rec["grid"] <= 8 * lim["sm_count"]
        else:
            assert rec["levels"][1]["span"] == S.ALL
            assert V & (V - 1) == 0 and 1 <= V <= 32 and chunk == 4 * (32 // V)
            assert rec["grid"] <= 4 * lim["sm_count"]
        assert rec["grid"] == min(rec["grid"], -(-N // chunk)) and (N == 0 or rec["grid"] >= 1)
        nodes = shape[2] if len(shape) == 3 else shape[0]
        assert rec["workspace_bytes"] >= 256 + 4 * nodes

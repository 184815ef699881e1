"""Pins for oracle/select.py: values printed in PAPER.md (tests/golden/paper_pins.json), the paper's
qualitative claims, and the DESIGN.md spec (Appendix-A style vectors, marked 'spec')."""
import itertools
import json
import os

import pytest

from oracle import select as S

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_pins.json")))
PAPER_SHAPES = [(65536, 1024), (8192, 8192), (1024, 65536)]


def _rec(pattern, shape, strategy="LITERAL", lim=S.B200, dtype="f32"):
    return S.select(pattern, shape, dtype, lim, strategy)


def _lv(r):
    return [(l["dim"], l["block"], l["span"], l["factor"]) for l in r["levels"]]


# ------------------------------------------------------------ Fig 6 (L450-452, L541, L549-550)

@pytest.mark.parametrize("M,N", [(192, 32), (640, 96), (1024, 4096)])
def test_fig6_blocks_and_dop(M, N):
    bx, by = GOLD["fig6"]["block"]["x"], GOLD["fig6"]["block"]["y"]
    # (a) Span(1) on both: M/64 x N/16 blocks, DOP M x N
    a_blocks = S.level_blocks(M, bx, S.ONE, 1) * S.level_blocks(N, by, S.ONE, 1)
    assert a_blocks == (M // 64) * (N // 16)
    assert S.level_dop(M, bx, S.ONE, 1) * S.level_dop(N, by, S.ONE, 1) == M * N
    # (b) Span(all) on x, Span(2) on y: N/32 blocks, DOP 64 x N/2 = 32N
    b_blocks = S.level_blocks(M, bx, S.ALL, 1) * S.level_blocks(N, by, S.SPAN_N, 2)
    assert b_blocks == N // 32
    assert S.level_dop(M, bx, S.ALL, 1) * S.level_dop(N, by, S.SPAN_N, 2) == 32 * N
    # (c) Split(3) on x, Span(2) on y: 3 x N/32 blocks, DOP x3 = 96N
    c_blocks = S.level_blocks(M, bx, S.SPLIT, 3) * S.level_blocks(N, by, S.SPAN_N, 2)
    assert c_blocks == 3 * N // 32
    assert S.level_dop(M, bx, S.SPLIT, 3) * S.level_dop(N, by, S.SPAN_N, 2) == 96 * N


# ------------------------------------------------------------ Fig 7 (L573-583)

@pytest.mark.parametrize("I,J", [(100, 50), (1024, 1024), (64, 4000), (65536, 1024), (8, 70000)])
def test_fig7_prior_mappings(I, J):
    tbt = _rec("SUM_ROWS", (I, J), "TB_T")
    assert [l["dim"] for l in tbt["levels"]] == [S.Y, S.X]
    assert tbt["levels"][0]["block"] == 1 and tbt["levels"][0]["span"] == S.ONE
    assert tbt["levels"][1]["span"] == S.ALL
    assert tbt["dop"] == I * min(J, GOLD["fig7"]["max_block_size"])
    warp = _rec("SUM_ROWS", (I, J), "WARP")
    assert [(l["dim"], l["block"]) for l in warp["levels"]] == [(S.Y, 16), (S.X, 32)]
    assert warp["dop"] == I * min(J, GOLD["fig7"]["warp_size"])


# ------------------------------------------------------------ ControlDOP constants (L799-803)

def test_k20c_min_max_dop():
    g = GOLD["controldop_k20c"]
    assert S.K20C["sm_count"] == g["sm_count"] and S.K20C["max_threads_per_sm"] == g["max_threads_per_sm"]
    assert S.min_max_dop(S.K20C) == (g["min_dop"], g["max_dop"])
    assert S.min_max_dop(S.B200) == (148 * 2048, 100 * 148 * 2048)


def test_search_space_base():
    g = GOLD["search_space"]
    assert S.SIZE_SET == g["sizeset"]
    assert len(g["dimset"]) * len(S.SIZE_SET) * len((S.ONE, S.ALL)) == g["base"] < 100


# ------------------------------------------------------------ hard constraints (Table II)

def test_hard_local_reduce_needs_span_all():
    nest = S.build_nest("SUM_ROWS", (100, 100))
    assert not S.hard_ok(nest, "f32", S.B200, (S.Y, S.X), (1, 64), (S.ONE, S.ONE))
    assert S.hard_ok(nest, "f32", S.B200, (S.Y, S.X), (1, 64), (S.ONE, S.ALL))


def test_hard_global_map_and_reduce_same_level():
    # LOGREG L2 holds a Map and a Reduce (dot): the level takes the conservative Span(all) (L655-656)
    r = _rec("LOGREG_GRAD", (16, 64, 256))
    assert r["levels"][2]["span"] == S.ALL


def test_fig9_mapping_is_infeasible():
    g = GOLD["fig9"]
    nest = S.build_nest("SUM_ROWS", (8192, 8192))
    assert 64 * 32 == g["threads"]
    assert not S.hard_ok(nest, "f32", S.B200, (S.Y, S.X), (64, 32), (S.ONE, S.ALL))
    assert S.hard_ok(nest, "f32", S.B200, (S.Y, S.X), (32, 32), (S.ONE, S.ALL))   # fails only by size


def test_hw_dim_limits():
    nest = S.build_nest("KMEANS_ASSIGN", (1000, 64, 32))
    # z is limited to 64 threads (max_block_dim)
    assert not S.hard_ok(nest, "f32", S.B200, (S.Y, S.Z, S.X), (1, 128, 8), (S.ONE, S.ALL, S.ALL))
    assert S.hard_ok(nest, "f32", S.B200, (S.Y, S.Z, S.X), (1, 16, 64), (S.ONE, S.ALL, S.ALL))


def test_register_and_smem_constraints_bind_on_tiny_device():
    tiny = dict(S.B200, regs_per_thread=128, smem_per_block=2048)
    nest = S.build_nest("SUM_ROWS", (1000, 1000))
    assert not S.hard_ok(nest, "f32", tiny, (S.Y, S.X), (1, 1024), (S.ONE, S.ALL))   # 128*1024 regs > 64K
    assert not S.hard_ok(nest, "f32", tiny, (S.Y, S.X), (1, 512), (S.ONE, S.ALL))    # 512*8 B smem > 2048
    assert S.hard_ok(nest, "f32", tiny, (S.Y, S.X), (1, 256), (S.ONE, S.ALL))
    r = _rec("SUM_ROWS", (1000, 1000), lim=tiny)
    assert r["levels"][1]["block"] == 256


# ------------------------------------------------------------ soft constraints / weights (Fig 8)

def test_fig8_inner_access_weight_dominates():
    I, J = 300, 500
    nest = S.build_nest("SUM_ROWS", (I, J))     # array1D(i) at L0, array2D(i,j) at L1 — Fig 8
    outer_x = S.score(nest, S.B200, (S.X, S.Y), (32, 32))
    inner_x = S.score(nest, S.B200, (S.Y, S.X), (32, 32))
    sg = I * J
    assert outer_x == S.W_C * I + sg            # α·I
    assert inner_x == S.W_C * I * J + sg        # α·I·J
    assert inner_x > outer_x


@pytest.mark.parametrize("shape", PAPER_SHAPES + [(1024, 1024), (100, 3000), (3000, 100)])
def test_coalescing_dims(shape):
    # sumCols assigns the outer (column) pattern to x; sumRows the inner one (L596-600, L1036-1044)
    assert _rec("SUM_COLS", shape)["levels"][0]["dim"] == S.X
    assert _rec("SUM_ROWS", shape)["levels"][1]["dim"] == S.X
    for strat in ("LITERAL", "AUTO"):
        r = _rec("SUM_COLS", shape, strat)
        assert r["levels"][0]["block"] * r["vec"] % 32 == 0 or shape[1] < 32


def test_split_only_on_sync_span_all_levels():
    for pat in ("SUM_ROWS", "SUM_COLS"):
        for R in (1, 7, 100, 1024, 4096, 65536, 1 << 20):
            for C in (1, 3, 64, 1000, 4096, 65536):
                if R * C > 1 << 32:
                    continue
                for lim in (S.B200, S.K20C):
                    nest = S.build_nest(pat, (R, C))
                    r = _rec(pat, (R, C), lim=lim)
                    for l, lv in enumerate(r["levels"]):
                        if lv["span"] == S.SPLIT:
                            assert nest["levels"][l][1]            # a Reduce level
                        if lv["span"] == S.SPAN_N:
                            assert not nest["levels"][l][1]


def test_search_is_the_argmax():
    # independent re-enumeration on small nests: no feasible candidate beats the chosen key
    for pat, shape in [("SUM_ROWS", (40, 70)), ("SUM_COLS", (70, 40)), ("SUM_COLS", (5, 3))]:
        nest = S.build_nest(pat, shape)
        dims, blocks, spans, sc = S.search(nest, "f32", S.B200)
        best = (sc, S.mapping_dop(nest, blocks, spans, [1, 1]), -blocks[0] * blocks[1])
        for d in itertools.permutations(range(2)):
            for b in itertools.product(S.SIZE_SET, repeat=2):
                for s in itertools.product((S.ONE, S.ALL), repeat=2):
                    if S.hard_ok(nest, "f32", S.B200, d, b, s):
                        key = (S.score(nest, S.B200, d, b), S.mapping_dop(nest, b, s, [1, 1]), -b[0] * b[1])
                        assert key <= best


def test_no_feasible_mapping():
    broken = dict(S.B200, max_threads_per_block=0)
    with pytest.raises(S.NoFeasibleMapping):
        _rec("SUM_ROWS", (10, 10), lim=broken)


# ------------------------------------------------------------ spec vectors (not paper values)

def test_spec_literal_vectors_b200():
    assert _lv(_rec("SUM_ROWS", (1024, 1024))) == [(S.Y, 1, S.ONE, 1), (S.X, 1024, S.ALL, 1)]
    assert _lv(_rec("SUM_ROWS", (65536, 1024))) == [(S.Y, 1, S.SPAN_N, 3), (S.X, 1024, S.ALL, 1)]
    assert _lv(_rec("SUM_ROWS", (1 << 20, 4096))) == [(S.Y, 1, S.SPAN_N, 36), (S.X, 1024, S.ALL, 1)]
    assert _lv(_rec("SUM_COLS", (65536, 1024))) == [(S.X, 32, S.ONE, 1), (S.Y, 32, S.SPLIT, 10)]
    assert _rec("SUM_COLS", (65536, 1024))["grid"] == 320
    assert _lv(_rec("SUM_COLS", (8192, 8192))) == [(S.X, 32, S.ONE, 1), (S.Y, 32, S.SPLIT, 2)]
    assert _lv(_rec("SUM_COLS", (1024, 65536))) == [(S.X, 32, S.ONE, 1), (S.Y, 32, S.ALL, 1)]
    assert _lv(_rec("SUM_COLS", (1 << 20, 4096))) == [(S.X, 32, S.ONE, 1), (S.Y, 32, S.SPLIT, 3)]
    assert _lv(_rec("KMEANS_ASSIGN", (1 << 22, 64, 32))) == [
        (S.Y, 1, S.SPAN_N, 142), (S.Z, 16, S.ALL, 1), (S.X, 64, S.ALL, 1)]
    assert _lv(_rec("LOGREG_GRAD", (4096, 4096, 256))) == [
        (S.Y, 1, S.ONE, 1), (S.Z, 4, S.ALL, 1), (S.X, 256, S.ALL, 1)]


def test_spec_literal_vectors_k20c():
    assert _lv(_rec("SUM_ROWS", (65536, 1024), lim=S.K20C))[0] == (S.Y, 1, S.SPAN_N, 26)
    assert _lv(_rec("SUM_ROWS", (8192, 8192), lim=S.K20C))[0] == (S.Y, 1, S.SPAN_N, 4)
    assert _lv(_rec("SUM_COLS", (65536, 1024), lim=S.K20C))[1] == (S.Y, 32, S.ALL, 1)


def test_spec_forced_1d():
    r = _rec("SUM_COLS", (65536, 1024), "1D")
    assert _lv(r) == [(S.X, 64, S.ONE, 1), (S.Y, 1, S.ALL, 1)] and r["dop"] == 1024 and r["grid"] == 16
    r = _rec("SUM_ROWS", (1024, 65536), "1D")
    assert _lv(r) == [(S.X, 64, S.ONE, 1), (S.Y, 1, S.ALL, 1)] and r["dop"] == 1024


# ------------------------------------------------------------ R2 invariants (S8)

@pytest.mark.parametrize("pat", ["SUM_ROWS", "SUM_COLS"])
@pytest.mark.parametrize("shape", PAPER_SHAPES + [(1, 1), (3, 5), (1000, 999), (1 << 20, 4096), (7, 100000)])
@pytest.mark.parametrize("dtype", ["f32", "i32", "i64"])
def test_r2_invariants(pat, shape, dtype):
    r = _rec(pat, shape, "AUTO", dtype=dtype)
    nest = S.build_nest(pat, shape)
    S_slots = S.slots(S.B200, S.T_BLOCK)
    assert r["grid"] <= S_slots and r["block"][0] * r["block"][1] == S.T_BLOCK
    for l, lv in enumerate(r["levels"]):
        n = nest["levels"][l][0]
        assert lv["grid"] == -(-n // lv["chunk"])
        if lv["dim"] == S.X and lv["span"] == S.SPLIT:
            assert lv["chunk"] % r["vec"] == 0
    assert r["vec"] in (1, 16 // S.DTYPE_SIZE[dtype])


# ---------------------------------------------------------------- NEXT rows: hand-computed records

def test_rowscols_regions_by_hand():
    # DESIGN.md S8 RC on B200 (S = 148): [8K,8K] f32 has Tr = 256 bands x Tc = 32 tiles; gc = 4 column
    # groups of 8 tiles and gr = 37 row regions of 7 bands give 148 regions of <= 56 tiles (the fair share
    # is 8192/148 = 55.35); [64K,1K]: 147 row regions of 14 bands, all 4 column tiles (rows written
    # directly); [1K,64K]: 4 x 37 regions of 8 bands x 7 tiles
    t = S.rc_tiling(8192, 8192, "f32", S.B200)
    assert (t["Tr"], t["Tc"], t["cr"], t["cc"], t["gr"], t["gc"], t["G"]) == (256, 32, 7, 8, 37, 4, 148)
    t = S.rc_tiling(65536, 1024, "f32", S.B200)
    assert (t["cr"], t["cc"], t["gr"], t["gc"], t["G"]) == (14, 4, 147, 1, 147)
    t = S.rc_tiling(1024, 65536, "f32", S.B200)
    assert (t["cr"], t["cc"], t["gr"], t["gc"], t["G"]) == (8, 7, 4, 37, 148)
    rec = S.select("SUM_ROWS_COLS", (8192, 8192), "f32", S.B200, "AUTO")
    assert rec["kernel_class"] == S.RC and rec["staged"] == 1 and rec["grid"] == 148
    assert [lv["span"] for lv in rec["levels"]] == [S.SPLIT, S.SPLIT]
    assert [lv["factor"] for lv in rec["levels"]] == [37, 4]
    assert [lv["chunk"] for lv in rec["levels"]] == [32 * 7, 256 * 8]
    # tickets [37] + [4] (256 B each), accumulators [8192] + [8192] fp64
    assert rec["workspace_bytes"] == 256 + 256 + 8192 * 8 + 8192 * 8


def test_kmeans_update_record_by_hand():
    # 4M points / 96 = 43691 tiles over 148 SMs: P = 296 tiles per block, G = ceil(43691/296) = 148;
    # workspace = 256-B ticket + 32 x 65 fp64 accumulators rounded up to 256 B
    rec = S.select("KMEANS_UPDATE", (1 << 22, 64, 32), "f32", S.B200, "AUTO")
    assert rec["kernel_class"] == S.KU and rec["grid"] == 148 and rec["claim_tiles"] == 296
    assert [lv["block"] for lv in rec["levels"]] == [12, 32]
    assert rec["levels"][0]["chunk"] == 96 * 296 and rec["levels"][0]["factor"] == 148
    assert rec["workspace_bytes"] == 256 + 256 * -(-32 * 65 * 8 // 256)


def test_pagerank_record_by_hand():
    # mean in-degree ceil(63710769 / 4194304) = 16 >= 8 -> segmented: 8 warps x 32 lanes, warp claims of 31
    # rows (ceil(4M / 31) = 135301 chunks), the chunk's edges Split over 32 lanes, min(8 x 148, 135301) =
    # 1184 blocks; workspace = claim counter + contrib [4M] f32
    rec = S.select("PAGERANK", (1 << 22, 63710769), "f32", S.B200, "AUTO")
    assert rec["kernel_class"] == S.PR and rec["staged"] == 0
    assert [lv["block"] for lv in rec["levels"]] == [8, 32]
    assert [lv["span"] for lv in rec["levels"]] == [S.SPAN_N, S.SPLIT]
    assert rec["levels"][0]["chunk"] == 31 and rec["levels"][0]["grid"] == -(-(1 << 22) // 31)
    assert rec["grid"] == 1184 and rec["claim_tiles"] == 31 and rec["levels"][1]["chunk"] == 16
    assert rec["workspace_bytes"] == 256 + 4 * (1 << 22)
    # mean in-degree 4 < 8 -> row groups: V = pow2 >= 4/4 = 1 lane per row, 256 row groups per block,
    # warp claims of 4 rows x 32 groups = 128 rows, min(4 x 148, 32768) = 592 blocks
    rec = S.select("PAGERANK", (1 << 22, 16443020), "f32", S.B200, "AUTO")
    assert [lv["block"] for lv in rec["levels"]] == [256, 1] and rec["levels"][1]["span"] == S.ALL
    assert rec["levels"][0]["chunk"] == 128 and rec["grid"] == 592 and rec["claim_tiles"] == 128

# ------------------------------------------------------------ readings the paper leaves open
# The paper fixes only that coalescing has the highest intrinsic weight (L674-676) and that equally good
# candidates are picked at random (L741). Any W_C > W_B and any tie-break are therefore valid readings;
# these tests pin that the records of every BASELINE.json workload do not depend on which one is taken.

BASELINE_CASES = [("SUM_ROWS", (1024, 1024)), ("SUM_COLS", (1024, 1024))] + \
    [(p, s) for s in PAPER_SHAPES for p in ("SUM_ROWS", "SUM_COLS")] + \
    [("SUM_COLS", (1 << 20, 4096)), ("KMEANS_ASSIGN", (1 << 22, 64, 32)), ("LOGREG_GRAD", (4096, 4096, 256)),
     ("SUM_ROWS_COLS", (8192, 8192)), ("SUM_WEIGHTED_ROWS", (8192, 8192)), ("SUM_WEIGHTED_COLS", (8192, 8192)),
     ("KMEANS_UPDATE", (1 << 22, 64, 32)), ("PAGERANK", (1 << 22, 63710769))]


def _records(strategies=("LITERAL", "AUTO")):
    out = {}
    for pat, shape in BASELINE_CASES:
        for strat in strategies:
            try:
                r = S.select(pat, shape, "f32", S.B200, strat)
                r = {k: v for k, v in r.items() if k != "score"}  # the score's scale is the weights'
            except S.Unsupported as e:
                r = ("unsupported", str(e))
            out[(pat, shape, strat)] = r
    return out


@pytest.mark.parametrize("w_c", [2, 3, 4, 16, 64, 1000])
def test_weight_reading_is_immaterial_on_the_baseline_workloads(monkeypatch, w_c):
    base = _records()
    monkeypatch.setattr(S, "W_C", w_c)   # any W_C > W_B = 1 honours "coalescing has the highest weight"
    assert _records() == base


def _tied_best(nest):
    """Every candidate of Algorithm 1's CandSet that attains the maximal (score, DOP) — the set the paper
    picks from at random (L741)."""
    L = len(nest["levels"])
    best, cands = None, []
    for dims in itertools.permutations(range(L)):
        for blocks in itertools.product(S.SIZE_SET, repeat=L):
            for spans in itertools.product((S.ONE, S.ALL), repeat=L):
                if not S.hard_ok(nest, "f32", S.B200, dims, blocks, spans):
                    continue
                key = (S.score(nest, S.B200, dims, blocks), S.mapping_dop(nest, blocks, spans, [1] * L))
                if best is None or key > best:
                    best, cands = key, []
                if key == best:
                    cands.append((tuple(dims), tuple(blocks), tuple(spans), key[0]))
    return cands


@pytest.mark.parametrize("pat,shape", [(p, s) for p, s in BASELINE_CASES if p in ("SUM_ROWS", "SUM_COLS")])
def test_sums_argmax_is_unique(pat, shape):
    # the headline sums: Algorithm 1's maximum is attained once, so no tie-break reading can change it
    assert len(_tied_best(S.build_nest(pat, shape))) == 1


@pytest.mark.parametrize("pat,shape", [("LOGREG_GRAD", (4096, 4096, 256)), ("KMEANS_ASSIGN", (1 << 16, 64, 32)),
                                       ("SUM_ROWS_COLS", (8192, 8192))])
def test_tie_break_reading_changes_no_auto_schedule(monkeypatch, pat, shape):
    # where several candidates tie, each one (as "the random pick") yields the same AUTO record up to which
    # of y / z carries the two non-x levels — a label the staged kernels do not read
    def norm(r):
        return ([(lv["block"], lv["span"], lv["factor"], lv["chunk"], lv["grid"], lv["dim"] == S.X)
                 for lv in r["levels"]], r["grid"], r["claim_tiles"], r["workspace_bytes"], r["staged"])
    cands = _tied_best(S.build_nest(pat, shape))
    assert len(cands) > 1
    recs = []
    for c in cands:
        monkeypatch.setattr(S, "search", lambda *a, _c=c, **k: _c)
        recs.append(norm(S.select(pat, shape, "f32", S.B200, "AUTO")))
    assert all(r == recs[0] for r in recs)

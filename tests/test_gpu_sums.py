"""GPU parity: the CUDA sum families (through the C-ABI) vs the fp64/int oracle, element by element.

Integers: bit-exact. fp32: |gpu - oracle| <= 1e-5 * Σ|terms| per output (north_star tolerance; for the
non-negative U[0,1) inputs this is 1e-5 relative). fp64: <= 1e-12 * Σ|terms|.
"""
import numpy as np
import pytest
import torch

from oracle import select as osel
from oracle import sums
from synth import gen

pytestmark = pytest.mark.gpu

STRATS = ["AUTO", "LITERAL", "1D", "TB_T", "WARP"]
SHAPES = [(1, 1), (3, 5), (31, 33), (33, 31), (1000, 999), (1024, 1024), (4097, 300), (300, 4097),
          (7, 70000), (70000, 7), (2, 1 << 17), (1001, 1024), (9, 3072)]


@pytest.fixture(scope="module")
def npp(cuda_device):
    from paper_conf_micro_leebsro14_b200 import npp as _npp
    return _npp


def _make(dtype, shape, seed, device):
    if dtype == "f32":
        return gen.uniform_f32(seed, shape, device=device)
    if dtype == "f64":
        return gen.uniform_f64(seed, shape, lo=-1.0, scale=2.0, device=device)  # signed: cancellation
    if dtype == "i32":
        return gen.int_uniform(seed, shape, -1000, 1000, device=device)
    return gen.int64_wide(seed, shape, device=device)


def _oracle(pattern, m_np):
    return sums.sum_rows(m_np) if pattern == "SUM_ROWS" else sums.sum_cols(m_np)


def _abs_scale(pattern, m_np):
    return sums.sum_abs_rows(m_np) if pattern == "SUM_ROWS" else sums.sum_abs_cols(m_np)


def check(pattern, m, got, dtype):
    m_np = m.cpu().numpy()
    want = _oracle(pattern, m_np)
    g = got.cpu().numpy()
    if dtype in ("f32", "f64"):
        tol = (1e-5 if dtype == "f32" else 1e-12) * _abs_scale(pattern, m_np)
        err = np.abs(g.astype(np.float64) - want)
        bad = np.nonzero(err > tol)[0]
        assert bad.size == 0, f"{pattern} first bad {bad[:5]} got {g[bad[:5]]} want {want[bad[:5]]}"
    else:
        assert np.array_equal(g.astype(np.int64), want.astype(np.int64)), pattern


@pytest.mark.parametrize("pattern", ["SUM_ROWS", "SUM_COLS"])
@pytest.mark.parametrize("dtype", ["f32", "i32", "i64", "f64"])
@pytest.mark.parametrize("strategy", STRATS)
def test_parity_small(npp, cuda_device, pattern, dtype, strategy):
    for i, shape in enumerate(SHAPES):
        m = _make(dtype, shape, 100 + i, cuda_device)
        p = npp.Plan(pattern, shape, dtype, strategy)
        out = p.new_out()
        p.execute([m], out)
        torch.cuda.synchronize()
        check(pattern, m, out, dtype)
        # the record the plan executes is the oracle selector's record (limits from the device)
        lim = npp.limits_query(0)
        assert p.mapping == osel.select(pattern, shape, dtype, lim, strategy)


@pytest.mark.parametrize("pattern", ["SUM_ROWS", "SUM_COLS"])
def test_exact_summable_fp32_bit_exact(npp, cuda_device, pattern):
    for shape in [(1024, 1024), (65536, 64), (64, 65536)]:
        m = gen.exact_f32(11, shape, device=cuda_device)
        for strategy in STRATS:
            p = npp.Plan(pattern, shape, "f32", strategy)
            out = p.execute([m], p.new_out())
            torch.cuda.synchronize()
            want = _oracle(pattern, m.cpu().numpy())
            assert np.array_equal(out.cpu().numpy().astype(np.float64), want), (shape, strategy)


def test_arange_int32_wrap(npp, cuda_device):
    shape = (3000, 2500)
    m = gen.arange_matrix(shape, torch.int32, offset=(1 << 31) - 10 ** 6, device=cuda_device)
    for pattern in ("SUM_ROWS", "SUM_COLS"):
        for strategy in STRATS:
            p = npp.Plan(pattern, shape, "i32", strategy)
            out = p.execute([m], p.new_out())
            torch.cuda.synchronize()
            check(pattern, m, out, "i32")


@pytest.mark.parametrize("shape", [(65536, 1024), (8192, 8192), (1024, 65536)])
def test_paper_shapes_full(npp, cuda_device, shape):
    m = gen.uniform_f32(3, shape, device=cuda_device)
    for pattern in ("SUM_ROWS", "SUM_COLS"):
        for strategy in STRATS:
            p = npp.Plan(pattern, shape, "f32", strategy)
            out = p.execute([m], p.new_out())
            out2 = p.execute([m], p.new_out())   # workspace reuse: tickets were reset
            torch.cuda.synchronize()
            check(pattern, m, out, "f32")
            # workspace reuse leaves no stale state; cut tiles add fp64 partials in arrival order, so
            # an fp32 output may differ by one ulp near a rounding tie (S8 staged note)
            assert torch.all((out - out2).abs() <= out.abs() * 2.0 ** -23), "stale workspace"


@pytest.mark.parametrize("dtype", ["f32", "i32", "i64", "f64"])
def test_overlap_back_to_back(npp, cuda_device, dtype):
    # npp_execute_ex(NPP_EXEC_OVERLAP): programmatic dependent launches back to back on one stream —
    # the same plan (shared workspace: pool counter, tickets, accumulators) and different plans.
    # Results equal the oracle's and every workspace ends zero (S8 balance rule).
    shapes = [(65536, 1024), (1024, 65536), (4097, 300), (300, 4100), (33, 1 << 16)]
    if dtype in ("i64", "f64"):
        shapes = [(s[0], s[1] // 2) if s[1] % 2 == 0 else s for s in shapes]
    plans = []
    for i, s in enumerate(shapes):
        m = _make(dtype, s, 40 + i, cuda_device)
        for pat in ("SUM_ROWS", "SUM_COLS"):
            plans.append((npp.Plan(pat, s, dtype, "AUTO"), m))
    outs = []
    for rep in range(3):
        for p, m in plans:
            outs.append((p, m, p.execute([m], p.new_out(), overlap=True)))
    torch.cuda.synchronize()
    for p, m, o in outs:
        check(p.pattern, m, o, dtype)
    for p, _ in plans:
        assert p.mapping["staged"] == 1
        assert int(p.workspace.count_nonzero()) == 0, p.shape


@pytest.mark.parametrize("pattern,shapes", [
    # SUM_ROWS, row pitch 64-256 KB and a multiple of 32 KB: one-row 32 KB tiles, whole rows (DESIGN S8 RX rule)
    ("SUM_ROWS", [(1024, 65536), (1000, 16384), (3, 65536), (4099, 24576), (1, 65536)]),
    # SUM_COLS, row pitch >= 64 KB and <= 1024 rows: MX-narrow strips, whole strips (DESIGN S8 MX-narrow rule)
    ("SUM_COLS", [(1024, 65536), (1000, 70000), (777, 16384), (129, 65536), (1, 1 << 20), (1024, 65540)]),
])
@pytest.mark.parametrize("dtype", ["f32", "i32", "i64"])
def test_large_pitch_whole_tile_rules(npp, cuda_device, pattern, shapes, dtype):
    # the large-pitch staged rules never cut a row / strip: back-to-back and PDL executes match the
    # oracle and leave the workspace (pool counter, tickets) zero
    for i, s in enumerate(shapes):
        if dtype == "i64" and s[1] % 2 == 0:
            s = (s[0], s[1] // 2)
        m = _make(dtype, s, 60 + i, cuda_device)
        p = npp.Plan(pattern, s, dtype)
        o1 = p.execute([m], p.new_out())
        o2 = p.execute([m], p.new_out(), overlap=True)
        torch.cuda.synchronize()
        check(pattern, m, o1, dtype)
        check(pattern, m, o2, dtype)
        assert int(p.workspace.count_nonzero()) == 0, (s, dtype)


@pytest.mark.parametrize("data", ["small_int", "uniform"])
def test_large_sumcols_full(npp, cuda_device, data):
    # BASELINE.json config 3: [1M, 4K] fp32 (16 GiB, 2^32 elements: 64-bit indexing). Every one of the
    # 4096 column sums and 1M row sums is compared with the oracle, which runs over 64K-row chunks
    # (exact for the integer-valued data; fp64 chunk sums for the U[0,1) data of the bench)
    R, C = 1 << 20, 4096
    free, _ = torch.cuda.mem_get_info()
    if free < 18 * (1 << 30):
        pytest.skip("needs 18 GiB free")
    m = (gen.small_int_f32(4, (R, C), 0, 15, device=cuda_device) if data == "small_int"
         else gen.uniform_f32(4, (R, C), device=cuda_device))
    p = npp.Plan("SUM_COLS", (R, C), "f32", "AUTO")
    out = p.execute([m], p.new_out())
    pr = npp.Plan("SUM_ROWS", (R, C), "f32", "AUTO")
    out_r = pr.execute([m], pr.new_out())
    torch.cuda.synchronize()
    got_c = out.cpu().numpy().astype(np.float64)
    got_r = out_r.cpu().numpy().astype(np.float64)
    want_c = np.zeros(C)
    scale_c = np.zeros(C)
    step = 1 << 16
    for r0 in range(0, R, step):
        chunk = m[r0:r0 + step].cpu().numpy()
        want_c += sums.sum_cols(chunk)
        scale_c += sums.sum_abs_cols(chunk)
        want_r = sums.sum_rows(chunk)
        if data == "small_int":
            assert np.array_equal(got_r[r0:r0 + step], want_r), r0
        else:
            assert np.all(np.abs(got_r[r0:r0 + step] - want_r) <= 1e-5 * sums.sum_abs_rows(chunk)), r0
    if data == "small_int":
        assert np.array_equal(got_c, want_c)
        assert float(out.double().sum()) == float(out_r.double().sum())
    else:
        assert np.all(np.abs(got_c - want_c) <= 1e-5 * scale_c)
    del m


def test_empty_and_degenerate(npp, cuda_device):
    p = npp.Plan("SUM_ROWS", (5, 0), "f32", "AUTO")
    out = torch.full((5,), 7.0, device=cuda_device)
    p.execute([torch.empty(0, device=cuda_device)], out)
    torch.cuda.synchronize()
    assert out.tolist() == [0.0] * 5
    p = npp.Plan("SUM_COLS", (0, 3), "i32", "AUTO")
    out = torch.full((3,), 7, dtype=torch.int32, device=cuda_device)
    p.execute([torch.empty(0, dtype=torch.int32, device=cuda_device)], out)
    torch.cuda.synchronize()
    assert out.tolist() == [0, 0, 0]
    p = npp.Plan("SUM_ROWS", (0, 3), "i32", "AUTO")
    assert p.launches == 0


def test_alignment_error(npp, cuda_device):
    base = gen.uniform_f32(1, (1024 * 1024 + 1,), device=cuda_device)
    m = base[1:].view(1024, 1024)
    p = npp.Plan("SUM_ROWS", (1024, 1024), "f32", "AUTO")
    assert p.mapping["vec"] == 4
    with pytest.raises(npp.NppError) as e:
        p.execute([m], p.new_out())
    assert e.value.status == npp.ERR_ALIGNMENT
    # the scalar literal mapping accepts it
    p1 = npp.Plan("SUM_ROWS", (1024, 1024), "f32", "TB_T")
    out = p1.execute([m], p1.new_out())
    torch.cuda.synchronize()
    check("SUM_ROWS", m, out, "f32")


def test_explicit_mappings(npp, cuda_device):
    # Fig 9's mapping (DimY 64 x DimX 32 = 2048 threads) is rejected by the hard constraints
    fig9 = dict(levels=[dict(dim=1, block=64, span=0), dict(dim=0, block=32, span=1)], vec=1)
    with pytest.raises(npp.NppError) as e:
        npp.Plan("SUM_ROWS", (8192, 8192), "f32", mapping=fig9)
    assert e.value.status == npp.ERR_NO_FEASIBLE
    # Split on a Map level is rejected
    bad = dict(levels=[dict(dim=1, block=8, span=3, factor=2), dict(dim=0, block=32, span=1)], vec=1)
    with pytest.raises(npp.NppError):
        npp.Plan("SUM_ROWS", (1000, 1000), "f32", mapping=bad)
    # the same mapping with 16 rows per block, Split(7) on the inner level, vector loads
    ok = dict(levels=[dict(dim=1, block=16, span=2, factor=3), dict(dim=0, block=32, span=3, factor=7)], vec=4)
    m = gen.uniform_f32(2, (1000, 1000), device=cuda_device)
    p = npp.Plan("SUM_ROWS", (1000, 1000), "f32", mapping=ok)
    assert p.mapping["levels"][1]["grid"] == 7 and p.workspace_bytes > 0
    for _ in range(3):
        out = p.execute([m], p.new_out())
    torch.cuda.synchronize()
    check("SUM_ROWS", m, out, "f32")
    # sumCols with y-outer/x-inner Split over rows (strided inner on x)
    m2 = gen.int_uniform(5, (5000, 300), -7, 7, device=cuda_device)
    mp = dict(levels=[dict(dim=1, block=4, span=0), dict(dim=0, block=64, span=3, factor=5)], vec=1)
    p = npp.Plan("SUM_COLS", (5000, 300), "i32", mapping=mp)
    out = p.execute([m2], p.new_out())
    torch.cuda.synchronize()
    check("SUM_COLS", m2, out, "i32")


def test_streams_and_concurrent_plans(npp, cuda_device):
    shapes = [(4096, 4096), (16384, 512)]
    ms = [gen.uniform_f32(20 + i, s, device=cuda_device) for i, s in enumerate(shapes)]
    streams = [torch.cuda.Stream() for _ in shapes]
    outs = []
    for m, s, st in zip(ms, shapes, streams):
        p = npp.Plan("SUM_COLS", s, "f32", "AUTO")
        outs.append((p, p.execute([m], p.new_out(), stream=st)))
    torch.cuda.synchronize()
    for m, (p, out) in zip(ms, outs):
        check("SUM_COLS", m, out, "f32")


def _counters(p):
    """The part of a plan's workspace every execute must leave zero (S9): all of a staged
    plan's (pool counters, tickets, accumulators); the tickets of a direct-load Split plan (its
    partials [G_1 x O] are written before they are read and keep their values)."""
    ws, m = p.workspace, p.mapping
    if m["staged"]:
        return ws
    acc = 4 if p.dtype == "i32" else 8
    part = -(-m["levels"][1]["grid"] * p.out_shape()[0] * acc // 256) * 256
    return ws[part:part + -(-4 * m["levels"][0]["grid"] // 256) * 256]


@pytest.mark.parametrize("dtype", ["f32", "i32", "i64", "f64"])
def test_weighted(npp, cuda_device, dtype):
    # sumWeightedRows / sumWeightedCols (Fig 15): AUTO runs the staged TMA family with v staged per
    # tile (narrow and wide tiles, ragged edges), the literal / prior-work mappings the direct family
    shapes = [(1000, 999), (4096, 4096), (37, 70000), (1001, 1024), (9, 3072), (70000, 36)]
    for shape in shapes:
        m = _make(dtype, shape, 7, cuda_device)
        for pattern, vlen in (("SUM_WEIGHTED_ROWS", shape[1]), ("SUM_WEIGHTED_COLS", shape[0])):
            v = _make(dtype, (vlen,), 8, cuda_device) if dtype != "f32" else \
                gen.uniform_f32(8, (vlen,), device=cuda_device, lo=-1.0, scale=2.0)
            mn, vn = m.cpu().numpy(), v.cpu().numpy()
            if pattern == "SUM_WEIGHTED_ROWS":
                want = sums.sum_weighted_rows(mn, vn)
                scale = np.abs(mn.astype(np.float64)) @ np.abs(vn.astype(np.float64))
            else:
                want = sums.sum_weighted_cols(mn, vn)
                scale = np.abs(vn.astype(np.float64)) @ np.abs(mn.astype(np.float64))
            for strategy in ("AUTO", "LITERAL", "1D", "TB_T", "WARP"):
                p = npp.Plan(pattern, shape, dtype, strategy)
                if strategy == "AUTO":
                    assert p.mapping["staged"] == int(shape[1] % (16 // np.dtype(mn.dtype).itemsize) == 0)
                out = p.execute([m, v], p.new_out())
                out2 = p.execute([m, v], p.new_out(), overlap=True)  # PDL back to back, same workspace
                torch.cuda.synchronize()
                for o in (out, out2):
                    g = o.cpu().numpy()
                    if dtype in ("f32", "f64"):
                        tol = 1e-5 if dtype == "f32" else 1e-12
                        assert np.all(np.abs(g - want) <= tol * scale), (pattern, shape, strategy)
                    else:
                        assert np.array_equal(g.astype(np.int64), want.astype(np.int64)), (pattern, shape, strategy)
                if p.workspace is not None and p.mapping["temp"] == 0:  # S10 temp regions are scratch
                    assert int(_counters(p).count_nonzero()) == 0


@pytest.mark.parametrize("dtype", ["f32", "i32"])
def test_weighted_temp_modes(npp, cuda_device, dtype):
    # S10 (§V-A, Fig 16): the LITERAL weighted sums materialise their zipWith in a preallocated
    # [outer x inner] buffer laid out for the mapping (Fig 11); the same mapping also runs with the
    # row-major buffer ("prealloc w/o layout opt") and with a device malloc per outer iteration
    for shape in [(1000, 999), (300, 4097), (4097, 300), (64, 65)]:
        m = _make(dtype, shape, 17, cuda_device)
        for pattern, vlen in (("SUM_WEIGHTED_ROWS", shape[1]), ("SUM_WEIGHTED_COLS", shape[0])):
            v = _make(dtype, (vlen,), 18, cuda_device) if dtype != "f32" else \
                gen.uniform_f32(18, (vlen,), device=cuda_device, lo=-1.0, scale=2.0)
            mn, vn = m.cpu().numpy(), v.cpu().numpy()
            rows = pattern == "SUM_WEIGHTED_ROWS"
            want = sums.sum_weighted_rows(mn, vn) if rows else sums.sum_weighted_cols(mn, vn)
            scale = (np.abs(mn.astype(np.float64)) @ np.abs(vn.astype(np.float64)) if rows
                     else np.abs(vn.astype(np.float64)) @ np.abs(mn.astype(np.float64)))
            lit = npp.Plan(pattern, shape, dtype, "LITERAL").mapping
            M, N = (shape[0], shape[1]) if rows else (shape[1], shape[0])   # outer, inner sizes
            outer_on_x = lit["levels"][0]["dim"] == 0
            assert lit["temp"] == npp.TEMP_PREALLOC
            assert lit["temp_stride"] == ([1, M] if outer_on_x else [N, 1])   # Fig 11b / 11a
            variants = [("layout", dict(lit)), ("rowmajor", dict(lit, temp_stride=[N, 1])),
                        ("malloc", dict(lit, temp=npp.TEMP_MALLOC, temp_stride=[0, 1]))]
            for name, rec in variants:
                p = npp.Plan(pattern, shape, dtype, mapping=rec)
                out = p.execute([m, v], p.new_out())
                torch.cuda.synchronize()
                g = out.cpu().numpy()
                if dtype == "f32":
                    assert np.all(np.abs(g - want) <= 1e-5 * scale), (pattern, shape, name)
                else:
                    assert np.array_equal(g.astype(np.int64), want.astype(np.int64)), (pattern, shape, name)
                ws = p.workspace
                if name == "malloc":
                    assert int(ws[-256:].count_nonzero()) == 0, "a device malloc returned NULL"
                elif p.mapping["levels"][1]["grid"] == 1:
                    # white box: the buffer holds t(o, i) = m·v at o*ts_o + i*ts_i (Fig 11)
                    tdt = {"f32": torch.float32, "i32": torch.int32}[dtype]
                    t = ws[:M * N * 4].view(tdt).cpu().numpy()
                    so, si = rec["temp_stride"]
                    for (o, i) in [(0, 0), (M - 1, N - 1), (M // 2, N // 3), (1 % M, 2 % N)]:
                        r, c = (o, i) if rows else (i, o)
                        if dtype == "f32":
                            prod = np.float32(mn[r, c]) * np.float32(vn[i])
                        else:
                            prod = np.int32((int(mn[r, c]) * int(vn[i]) + (1 << 31)) % (1 << 32) - (1 << 31))
                        assert t[o * so + i * si] == prod, (pattern, shape, name, o, i)


RC_SHAPES = [(1, 1), (3, 5), (31, 33), (33, 31), (1000, 999), (1024, 1024), (4097, 300), (300, 4097),
             (7, 70000), (70000, 7), (2, 1 << 17), (1001, 1024), (9, 3072), (5000, 8192), (100000, 36),
             (3, 1 << 21), (40, 1200004)]   # more column groups than SMs: blocks walk several regions


def _check_rc(m, got, dtype):
    """SUM_ROWS_COLS output = [sumRows | sumCols] (S8 RC), each half to the sums' bar."""
    R = m.shape[0]
    check("SUM_ROWS", m, got[:R], dtype)
    check("SUM_COLS", m, got[R:], dtype)


@pytest.mark.parametrize("dtype", ["f32", "i32", "i64", "f64"])
def test_rows_cols_parity(npp, cuda_device, dtype):
    # one pass, both outputs: staged (16-B row pitch) and direct (ragged pitch) variants, regions cut
    # along rows only, columns only and both (tickets), ragged edge tiles; back-to-back executes
    # (plain and PDL-overlapped) on one workspace leave it zero
    lim = npp.limits_query(0)
    for i, shape in enumerate(RC_SHAPES):
        m = _make(dtype, shape, 300 + i, cuda_device)
        p = npp.Plan("SUM_ROWS_COLS", shape, dtype, "AUTO")
        assert p.mapping == osel.select("SUM_ROWS_COLS", shape, dtype, lim, "AUTO")
        assert p.mapping["kernel_class"] == npp.CLASS_RC
        assert p.mapping["staged"] == int(shape[1] % (16 // np.dtype(m.cpu().numpy().dtype).itemsize) == 0)
        outs = [p.execute([m], p.new_out()), p.execute([m], p.new_out(), overlap=True),
                p.execute([m], p.new_out())]
        torch.cuda.synchronize()
        for o in outs:
            _check_rc(m, o, dtype)
        assert int(p.workspace.count_nonzero()) == 0, shape


def test_rows_cols_exact_and_wrap(npp, cuda_device):
    # exact-summable fp32 makes both halves bit-exact; int32 arange wraps mod 2^32 in both directions
    for shape in [(1024, 1024), (65536, 64), (64, 65536)]:
        m = gen.exact_f32(11, shape, device=cuda_device)
        o = npp.Plan("SUM_ROWS_COLS", shape, "f32").execute([m], torch.empty(sum(shape), device=cuda_device))
        torch.cuda.synchronize()
        assert np.array_equal(o.cpu().numpy().astype(np.float64), sums.sum_rows_cols(m.cpu().numpy())), shape
    shape = (3000, 2500)
    m = gen.arange_matrix(shape, torch.int32, offset=(1 << 31) - 10 ** 6, device=cuda_device)
    o = npp.Plan("SUM_ROWS_COLS", shape, "i32").execute(
        [m], torch.empty(sum(shape), dtype=torch.int32, device=cuda_device))
    torch.cuda.synchronize()
    _check_rc(m, o, "i32")


@pytest.mark.parametrize("shape", [(65536, 1024), (8192, 8192), (1024, 65536)])
def test_rows_cols_paper_shapes(npp, cuda_device, shape):
    m = gen.uniform_f32(3, shape, device=cuda_device)
    rows, cols = npp.sum_rows_cols(m)
    torch.cuda.synchronize()
    check("SUM_ROWS", m, rows, "f32")
    check("SUM_COLS", m, cols, "f32")
    # the fused pass agrees with the two single-pattern plans
    r2, c2 = npp.sum_rows(m), npp.sum_cols(m)
    torch.cuda.synchronize()
    assert torch.all((rows - r2).abs() <= r2.abs() * 2.0 ** -22)
    assert torch.all((cols - c2).abs() <= c2.abs() * 2.0 ** -22)


def test_rows_cols_plan_rules(npp, cuda_device):
    # the one-pass family is AUTO only; the empty nest zero-fills both halves
    for strategy in ("LITERAL", "1D", "TB_T", "WARP"):
        with pytest.raises(npp.NppError) as e:
            npp.Plan("SUM_ROWS_COLS", (64, 64), "f32", strategy)
        assert e.value.status == npp.ERR_UNSUPPORTED
    for shape in [(0, 5), (7, 0)]:
        p = npp.Plan("SUM_ROWS_COLS", shape, "i32")
        o = p.execute([torch.empty(shape, dtype=torch.int32, device=cuda_device)],
                      torch.full((sum(shape),), 7, dtype=torch.int32, device=cuda_device))
        torch.cuda.synchronize()
        assert int(o.abs().sum()) == 0


@pytest.mark.parametrize("pattern", ["SUM_ROWS", "SUM_COLS", "SUM_WEIGHTED_ROWS", "SUM_WEIGHTED_COLS"])
def test_every_enumerated_mapping_executes_correctly(npp, cuda_device, pattern):
    # the Fig 17 space: every hard-feasible Algorithm 1 candidate that npp_enumerate lists
    # runs through npp_plan_with_mapping and matches the oracle, at two small shapes per nest (a ragged
    # one and a skewed one in the spirit of the paper's (50, 20K))
    lim = npp.limits_query(0)
    rows = pattern in ("SUM_ROWS", "SUM_WEIGHTED_ROWS")
    weighted = "WEIGHTED" in pattern
    for shape, dtype in [((97, 1003), "i32"), ((50, 20000), "f32")]:
        m = _make(dtype, shape, 61, cuda_device)
        v = _make(dtype, (shape[1] if rows else shape[0],), 62, cuda_device) if weighted else None
        m_np = m.cpu().numpy()
        if weighted:
            v_np = v.cpu().numpy()
            want = (sums.sum_weighted_rows(m_np, v_np) if rows else sums.sum_weighted_cols(m_np, v_np))
        else:
            want = _oracle("SUM_ROWS" if rows else "SUM_COLS", m_np)
        recs = npp.enumerate_mappings(pattern, shape, dtype, lim)
        assert len(recs) > 50
        for rec in recs:
            p = npp.Plan(pattern, shape, dtype, mapping=rec)
            out = p.execute([m, v] if weighted else [m], p.new_out())
            torch.cuda.synchronize()
            g = out.cpu().numpy()
            if dtype == "f32":
                scale = np.abs(want) if not weighted else None
                if weighted:
                    a_np = np.abs(m_np.astype(np.float64)) * (np.abs(v_np.astype(np.float64))[None, :] if rows
                                                               else np.abs(v_np.astype(np.float64))[:, None])
                    scale = a_np.sum(1) if rows else a_np.sum(0)
                assert np.all(np.abs(g.astype(np.float64) - want) <= 1e-5 * scale), rec["levels"]
            else:
                assert np.array_equal(g.astype(np.int64), np.asarray(want).astype(np.int64)), rec["levels"]

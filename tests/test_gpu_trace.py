"""GPU white-box test of the runtime rule R2 (S8): npp_execute_traced records which block
loaded each tile, and the schedule the kernels actually ran is compared with the one the mapping record
prescribes (tests/schedule.py, derived from the record's grid / claim_tiles / static_tiles / chunks):

  * every tile (region) is loaded exactly once;
  * staged sums: tiles of the static part belong to the block whose static range holds them; every
    claim-pool unit is streamed by one block; each block takes part;
  * LOGREG_GRAD / KMEANS_ASSIGN / KMEANS_UPDATE: tile t belongs to block t // claim_tiles;
  * SUM_ROWS_COLS: region q belongs to the block whose region range holds it;
and the traced execute still returns the oracle's result.
"""
import numpy as np
import pytest
import torch

from oracle import kmeans as okm
from oracle import logreg as olr
from oracle import sums
from schedule import contiguous_ranges, pool_units, rc_regions, staged_geometry, static_ranges
from synth import gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def npp(cuda_device):
    from paper_conf_micro_leebsro14_b200 import npp as _npp
    return _npp


def _owners(ranges, n):
    own = np.full(n, -1, dtype=np.int64)
    for b, (s0, s1) in enumerate(ranges):
        own[s0:s1] = b
    return own


SUM_CASES = [("SUM_ROWS", (65536, 1024)), ("SUM_ROWS", (8192, 8192)), ("SUM_ROWS", (1024, 65536)),
             ("SUM_COLS", (65536, 1024)), ("SUM_COLS", (8192, 8192)), ("SUM_COLS", (1024, 65536)),
             ("SUM_ROWS", (1000, 999 * 4)), ("SUM_COLS", (4097, 300)), ("SUM_COLS", (300, 4096)),
             ("SUM_ROWS", (3, 256 * 1024)), ("SUM_COLS", (129, 65536))]


@pytest.mark.parametrize("pattern,shape", SUM_CASES)
@pytest.mark.parametrize("dtype", ["f32", "i64"])
def test_staged_sum_schedule(npp, cuda_device, pattern, shape, dtype):
    m = (gen.uniform_f32(41, shape, device=cuda_device) if dtype == "f32"
         else gen.int64_wide(41, shape, device=cuda_device))
    p = npp.Plan(pattern, shape, dtype, "AUTO")
    rec = p.mapping
    assert rec["staged"] == 1
    To, Ti, BR, W, align = staged_geometry(pattern, shape, dtype, rec)
    T, G, U, Ts = To * Ti, rec["grid"], rec["claim_tiles"], rec["static_tiles"]
    assert p.tiles == T
    out = p.new_out()
    for rep in range(2):  # the second execute reuses the workspace the first left zeroed
        blk, cnt = p.execute_traced([m], out)
        torch.cuda.synchronize()
        blk, cnt = blk.cpu().numpy(), cnt.cpu().numpy()
        assert np.all(cnt == 1), f"tiles loaded != once: {np.nonzero(cnt != 1)[0][:8]}"
        own = _owners(static_ranges(G, Ts, Ti, align), T)
        assert np.array_equal(blk[:Ts], own[:Ts]), "static part differs from the record's ranges"
        for s0, s1 in pool_units(T, Ts, U, Ti, G):
            assert len(set(blk[s0:s1].tolist())) == 1, "a pool unit was split between blocks"
        ranges = static_ranges(G, Ts, Ti, align)
        # every block with static tiles takes part (blocks with an empty static range may find the
        # pool already drained: small shapes with Ts < G)
        assert {b for b, (s0, s1) in enumerate(ranges) if s1 > s0} <= set(blk.tolist())
        m_np = m.cpu().numpy()
        want = sums.sum_rows(m_np) if pattern == "SUM_ROWS" else sums.sum_cols(m_np)
        got = out.cpu().numpy()
        if dtype == "f32":
            scale = sums.sum_abs_rows(m_np) if pattern == "SUM_ROWS" else sums.sum_abs_cols(m_np)
            assert np.all(np.abs(got.astype(np.float64) - want) <= 1e-5 * scale)
        else:
            assert np.array_equal(got.astype(np.int64), want.astype(np.int64))


def _check_contiguous(blk, cnt, rec, T):
    assert np.all(cnt == 1)
    own = _owners(contiguous_ranges(T, rec["claim_tiles"], rec["grid"]), T)
    assert np.array_equal(blk, own)


def test_logreg_schedule(npp, cuda_device):
    for B, Rb, C in [(37, 1000, 256), (3, 4096, 64), (300, 64, 12)]:
        x, y, w = gen.logreg_inputs(B, Rb, C, seed=8, device=cuda_device)
        p = npp.Plan("LOGREG_GRAD", (B, Rb, C), "f32", "AUTO")
        T = B * (-(-Rb // 32))
        assert p.tiles == T
        out = p.new_out()
        blk, cnt = p.execute_traced([x, y, w], out)
        torch.cuda.synchronize()
        _check_contiguous(blk.cpu().numpy(), cnt.cpu().numpy(), p.mapping, T)
        xn, yn, wn = x.cpu().numpy(), y.cpu().numpy(), w.cpu().numpy()
        scale, _ = olr.grad_scales(xn, yn, wn, B)
        err = np.abs(out.cpu().numpy().astype(np.float64) - olr.grad(xn, yn, wn, B))
        assert np.all(err <= 1e-5 * scale)


def test_kmeans_schedule(npp, cuda_device):
    for N, D, K in [(100000, 64, 32), (5000, 128, 40), (300, 16, 5)]:
        x, c = gen.kmeans_inputs(N, D, K, device=cuda_device, integer=True)
        p = npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", "AUTO")
        TP = 256 if D <= 64 else 128
        T = -(-N // TP)
        assert p.tiles == T
        out = p.new_out()
        blk, cnt = p.execute_traced([x, c], out)
        torch.cuda.synchronize()
        _check_contiguous(blk.cpu().numpy(), cnt.cpu().numpy(), p.mapping, T)
        assert np.array_equal(out.cpu().numpy(), okm.assign(x.cpu().numpy(), c.cpu().numpy()))


def test_kmeans_update_schedule(npp, cuda_device):
    for N, D, K in [(200000, 64, 32), (1000, 8, 3)]:
        x, c = gen.kmeans_inputs(N, D, K, device=cuda_device, integer=True)
        keys = gen.int_uniform(9, (N,), 0, K - 1, dtype=torch.int32, device=cuda_device)
        p = npp.Plan("KMEANS_UPDATE", (N, D, K), "f32", "AUTO")
        T = -(-N // 96)  # DESIGN.md S8 KU: 96-point tiles
        assert p.tiles == T
        out = p.new_out()
        blk, cnt = p.execute_traced([x, keys], out)
        torch.cuda.synchronize()
        _check_contiguous(blk.cpu().numpy(), cnt.cpu().numpy(), p.mapping, T)
        want = okm.update(x.cpu().numpy(), keys.cpu().numpy(), K)
        assert np.array_equal(out.cpu().numpy().astype(np.float64), want)  # integer coordinates: exact


def test_rowscols_schedule(npp, cuda_device):
    for shape in [(65536, 1024), (8192, 8192), (1024, 65536), (1000, 3000)]:
        m = gen.int_uniform(12, shape, -1000, 1000, device=cuda_device)
        p = npp.Plan("SUM_ROWS_COLS", shape, "i32", "AUTO")
        gr, gc, nreg, G, ranges = rc_regions(p.mapping)
        assert p.tiles == nreg
        out = p.new_out()
        blk, cnt = p.execute_traced([m], out)
        torch.cuda.synchronize()
        blk, cnt = blk.cpu().numpy(), cnt.cpu().numpy()
        assert np.all(cnt == 1)
        assert np.array_equal(blk, _owners(ranges, nreg))
        m_np = m.cpu().numpy()
        want = np.concatenate([sums.sum_rows(m_np), sums.sum_cols(m_np)]).astype(np.int64)
        assert np.array_equal(out.cpu().numpy().astype(np.int64), want)


def test_traced_rejects_untiled_plans(npp, cuda_device):
    p = npp.Plan("SUM_ROWS", (100, 100), "f32", "LITERAL")
    assert p.tiles == 0
    m = gen.uniform_f32(1, (100, 100), device=cuda_device)
    with pytest.raises(npp.NppError) as e:
        p.execute_traced([m], p.new_out())
    assert e.value.status == npp.ERR_UNSUPPORTED

"""Seeded random-shape sweep of every AUTO family against the oracle (integers bit-exact, fp32 within
the DESIGN.md §5 bounds): shapes drawn to hit ragged tiles, single rows/columns, Split regions cut both
ways and more regions than SMs."""
import numpy as np
import pytest
import torch

from oracle import kmeans as okm
from oracle import pagerank as opr
from oracle import sums
from synth import gen

pytestmark = pytest.mark.gpu

RNG = np.random.default_rng(20261017)
SUM_SHAPES = [(int(RNG.integers(1, 3000)), int(RNG.integers(1, 3000))) for _ in range(24)] + \
             [(int(RNG.integers(1, 40)), int(RNG.integers(1, 200000))) for _ in range(6)] + \
             [(int(RNG.integers(1, 200000)), int(RNG.integers(1, 40))) for _ in range(6)]


@pytest.fixture(scope="module")
def npp(cuda_device):
    from paper_conf_micro_leebsro14_b200 import npp as _npp
    return _npp


def _mat(dtype, shape, seed, dev):
    if dtype == "f32":
        return gen.uniform_f32(seed, shape, device=dev)
    if dtype == "f64":
        return gen.uniform_f64(seed, shape, lo=-1.0, scale=2.0, device=dev)
    if dtype == "i32":
        return gen.int_uniform(seed, shape, -1000, 1000, device=dev)
    return gen.int64_wide(seed, shape, device=dev)


def _close(got, want, scale, dtype):
    if dtype in ("f32", "f64"):
        return np.all(np.abs(got.astype(np.float64) - want) <= (1e-5 if dtype == "f32" else 1e-12) * scale)
    return np.array_equal(got.astype(np.int64), want.astype(np.int64))


@pytest.mark.parametrize("dtype", ["f32", "i32", "i64", "f64"])
def test_random_sums_and_rows_cols(npp, cuda_device, dtype):
    for i, shape in enumerate(SUM_SHAPES):
        m = _mat(dtype, shape, 900 + i, cuda_device)
        mn = m.cpu().numpy()
        r, c = npp.sum_rows(m), npp.sum_cols(m)
        rc = npp.Plan("SUM_ROWS_COLS", shape, dtype).execute([m], torch.empty(sum(shape), dtype=m.dtype,
                                                                               device=cuda_device))
        torch.cuda.synchronize()
        wr, wc = sums.sum_rows(mn), sums.sum_cols(mn)
        sr, sc = sums.sum_abs_rows(mn), sums.sum_abs_cols(mn)
        for got, want, scale, name in ((r, wr, sr, "rows"), (c, wc, sc, "cols"), (rc[:shape[0]], wr, sr, "rc rows"),
                                       (rc[shape[0]:], wc, sc, "rc cols")):
            assert _close(got.cpu().numpy(), want, scale, dtype), (name, shape, dtype)


def test_random_kmeans_update(npp, cuda_device):
    for i in range(16):
        D = int(RNG.choice([4, 8, 12, 16, 32, 60, 64]))
        K = int(RNG.integers(1, max(2, min(256, 2048 // D))))
        N = int(RNG.integers(1, 40000))
        x, _ = gen.kmeans_inputs(N, D, K, seed=950 + i, device=cuda_device)
        a = gen.int_uniform(960 + i, (N,), -1, K, device=cuda_device)
        u = npp.kmeans_update(x, a, K)
        torch.cuda.synchronize()
        xn, an = x.cpu().numpy(), a.cpu().numpy()
        want, scale = okm.update(xn, an, K), okm.update_scale(xn, an, K)
        got = u.cpu().numpy().astype(np.float64)
        assert np.array_equal(got[:, -1], want[:, -1]), (N, D, K)
        assert np.all(np.abs(got[:, :-1] - want[:, :-1]) <= 1e-5 * scale + 1e-30), (N, D, K)


def test_random_pagerank(npp, cuda_device):
    for i in range(10):
        N = int(RNG.integers(1, 60000))
        avg = int(RNG.integers(1, 60))
        cap = int(RNG.integers(1, 3000))
        rp, ci, pr, od = gen.pagerank_inputs(N, avg_deg=avg, seed=970 + i, max_deg=cap, device=cuda_device)
        out = npp.pagerank_step(rp, ci, pr, od)
        torch.cuda.synchronize()
        want = opr.step(rp.cpu().numpy(), ci.cpu().numpy(), pr.cpu().numpy(), od.cpu().numpy())
        assert np.all(np.abs(out.cpu().numpy() - want) <= 1e-5 * want), (N, avg, cap)

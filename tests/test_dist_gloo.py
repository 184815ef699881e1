"""World-size-2 gloo tests of the multi-GPU sharding / reduction logic on CPU.

The kernels are replaced by a CPU stand-in through the `compute` hook (test infrastructure only), so
these tests check what the dist layer owns: shard ranges, shard-invariant inputs, and where the
collective sits (sumCols and the full-batch logreg reduce; sumRows / k-means / mini-batch logreg
do not).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import kmeans as okm
from oracle import logreg as olr
from oracle import sums
from paper_conf_micro_leebsro14_b200.dist import shard_range
from synth import gen

WORLD = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _cpu_rows(m):
    return torch.from_numpy(sums.sum_rows(m.numpy()))


def _cpu_cols(m):
    return torch.from_numpy(sums.sum_cols(m.numpy()))


def _worker(rank, port, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    from paper_conf_micro_leebsro14_b200 import dist as ndist
    try:
        R, C = 1001, 37
        lo, hi = shard_range(R, WORLD, rank)
        local = gen.uniform_f32(4, (hi - lo, C), offset=lo * C)
        cols = ndist.sum_cols(local, compute=_cpu_cols)                     # all-reduced column sums
        rows = ndist.sum_rows(local, gather=True, compute=_cpu_rows)        # gathered row sums
        li = gen.int_uniform(5, (hi - lo, C), -1000, 1000, offset=lo * C)
        cols_i = ndist.sum_cols(li.to(torch.int64), compute=lambda m: torch.from_numpy(sums.sum_cols(m.numpy())))
        # k-means: points sharded, centroids replicated
        N, D, K = 301, 8, 5
        plo, phi = shard_range(N, WORLD, rank)
        xs, c = gen.kmeans_inputs(phi - plo, D, K, row_offset=plo)
        a = ndist.kmeans_assign(xs, c, compute=lambda x, cc: torch.from_numpy(okm.assign(x.numpy(), cc.numpy())))
        # k-means update: each rank's [K, D+1] partial over its points, one all-reduce
        u = ndist.kmeans_update(xs, a, K, compute=lambda x, aa, k: torch.from_numpy(okm.update(x.numpy(), aa.numpy(), k)))
        # logreg full batch: rows sharded, one all-reduce of C floats
        Rb, Cl = 200, 12
        rlo, rhi = shard_range(Rb, WORLD, rank)
        xl, yl, w = gen.logreg_inputs(1, Rb, Cl, seed=6)
        g = ndist.logreg_grad(xl[rlo:rhi].contiguous(), yl[rlo:rhi].contiguous(), w, 1, full_batch=True,
                              compute=lambda x, y, ww, B: torch.from_numpy(olr.grad(x.numpy(), y.numpy(), ww.numpy(), B)))
        # PageRank: node rows sharded, pr / outdeg replicated, one all-gather of the next vector
        from oracle import pagerank as opr
        rp, ci, prv, od = gen.pagerank_inputs(501, avg_deg=6, seed=9, max_deg=64)
        nlo, nhi = shard_range(501, WORLD, rank)
        lrp = rp[nlo:nhi + 1] - rp[nlo]
        lci = ci[int(rp[nlo]):int(rp[nhi])]

        prn = ndist.pagerank_step(lrp, lci, prv, od, compute=lambda lr, lc, p, d, a0, a1: torch.from_numpy(
            opr.step(lr.numpy(), lc.numpy(), p.numpy(), d.numpy())))
        results[rank] = dict(cols=cols.numpy(), rows=rows.numpy(), cols_i=cols_i.numpy(), a=a.numpy(),
                             u=u.numpy(), g=g.numpy(), pr=prn.numpy(), lo=lo, hi=hi)
    finally:
        dist.destroy_process_group()


def test_shard_range_partitions():
    for n in (0, 1, 7, 1000, 1 << 20):
        for world in (1, 2, 3, 8):
            parts = [shard_range(n, world, r) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(parts[i][1] == parts[i + 1][0] for i in range(world - 1))
            sizes = [b - a for a, b in parts]
            assert max(sizes) - min(sizes) <= 1


def test_two_rank_gloo():
    port = _free_port()
    manager = mp.Manager()
    results = manager.dict()
    mp.start_processes(_worker, args=(port, results), nprocs=WORLD, join=True, start_method="spawn")
    R, C = 1001, 37
    full = gen.uniform_f32(4, (R, C)).numpy()
    want_cols = sums.sum_cols(full)
    want_rows = sums.sum_rows(full)
    fi = gen.int_uniform(5, (R, C), -1000, 1000).numpy().astype(np.int64)
    for rank in range(WORLD):
        r = results[rank]
        assert np.allclose(r["cols"], want_cols, rtol=1e-12)        # cross-rank Split(P) of the Reduce
        assert np.allclose(r["rows"], want_rows, rtol=1e-12)
        assert r["cols_i"].tolist() == sums.sum_cols(fi).tolist()   # integer reduce is exact
    a = np.concatenate([results[r]["a"] for r in range(WORLD)])
    x, c = gen.kmeans_inputs(301, 8, 5)
    assert a.tolist() == okm.assign(x.numpy(), c.numpy()).tolist()
    want_u = okm.update(x.numpy(), a, 5)
    for rank in range(WORLD):
        assert np.allclose(results[rank]["u"], want_u, rtol=1e-12, atol=1e-9)
        assert results[rank]["u"][:, -1].tolist() == want_u[:, -1].tolist()
    from oracle import pagerank as opr
    rp, ci, prv, od = gen.pagerank_inputs(501, avg_deg=6, seed=9, max_deg=64)
    want_pr = opr.step(rp.numpy(), ci.numpy(), prv.numpy(), od.numpy())
    for rank in range(WORLD):
        assert np.allclose(results[rank]["pr"], want_pr, rtol=1e-12)
    xl, yl, w = gen.logreg_inputs(1, 200, 12, seed=6)
    want_g = olr.grad(xl.numpy(), yl.numpy(), w.numpy(), 1)
    for rank in range(WORLD):
        assert np.allclose(results[rank]["g"], want_g, rtol=1e-12, atol=1e-12)

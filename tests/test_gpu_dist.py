"""GPU checks of the multi-GPU path on one device: a world-size-1 NCCL group through dist.*, and a
'fake multi-GPU' run that executes P row shards one after another on the same GPU and reduces them
(the same Split(P) the NCCL reduce performs across GPUs)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

from oracle import sums
from synth import gen

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.fixture(scope="module")
def nccl_group(cuda_device):
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ["MASTER_PORT"] = str(_free_port())
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=cuda_device)
    yield
    dist.destroy_process_group()


def test_nccl_world1_sum_cols_and_logreg(nccl_group, cuda_device):
    from paper_conf_micro_leebsro14_b200 import dist as ndist
    m = gen.uniform_f32(4, (70000, 300), device=cuda_device)
    cols = ndist.sum_cols(m)
    torch.cuda.synchronize()
    want = sums.sum_cols(m.cpu().numpy())
    assert np.allclose(cols.cpu().numpy(), want, rtol=1e-5)
    from oracle import logreg as olr
    x, y, w = gen.logreg_inputs(1, 4096, 256, device=cuda_device)
    g = ndist.logreg_grad(x, y, w, 1, full_batch=True)
    torch.cuda.synchronize()
    assert g.shape == (1, 256)
    xn, yn, wn = x.cpu().numpy(), y.cpu().numpy(), w.cpu().numpy()
    scale, _ = olr.grad_scales(xn, yn, wn, 1)
    assert np.all(np.abs(g.cpu().numpy().astype(np.float64) - olr.grad(xn, yn, wn, 1)) <= 1e-5 * scale)


@pytest.mark.parametrize("P", [2, 4, 8])
def test_fake_multigpu_row_shards(cuda_device, P):
    from paper_conf_micro_leebsro14_b200 import npp
    from paper_conf_micro_leebsro14_b200.dist import shard_range
    R, C = 1 << 17, 4096
    parts_c, parts_r = [], []
    for rank in range(P):
        lo, hi = shard_range(R, P, rank)
        shard = gen.small_int_f32(4, (hi - lo, C), 0, 15, offset=lo * C, device=cuda_device)
        parts_c.append(npp.sum_cols(shard).double())
        parts_r.append(npp.sum_rows(shard))
    torch.cuda.synchronize()
    full = gen.small_int_f32(4, (R, C), 0, 15).numpy()
    assert np.array_equal(sum(p for p in parts_c).cpu().numpy(), sums.sum_cols(full))   # exact data
    assert np.array_equal(torch.cat(parts_r).double().cpu().numpy(), sums.sum_rows(full))


def test_nccl_world1_kmeans_update_and_pagerank(nccl_group, cuda_device):
    # the NEXT rows' exchange steps through NCCL (world 1): the k-means update all-reduce and the
    # PageRank all-gather of the next vector, against the oracle
    from oracle import kmeans as okm
    from oracle import pagerank as opr
    from paper_conf_micro_leebsro14_b200 import dist as ndist
    x, _ = gen.kmeans_inputs(20000, 64, 32, device=cuda_device)
    a = gen.int_uniform(6, (20000,), 0, 31, device=cuda_device)
    u = ndist.kmeans_update(x, a, 32)
    torch.cuda.synchronize()
    want = okm.update(x.cpu().numpy(), a.cpu().numpy(), 32)
    assert np.array_equal(u.cpu().numpy()[:, -1], want[:, -1])
    scale = okm.update_scale(x.cpu().numpy(), a.cpu().numpy(), 32)  # 1e-5 Σ_{a_i=k} |x_id|
    assert np.all(np.abs(u.cpu().numpy()[:, :-1].astype(np.float64) - want[:, :-1]) <= 1e-5 * scale)
    rp, ci, pr, od = gen.pagerank_inputs(30000, avg_deg=10, seed=8, max_deg=500, device=cuda_device)
    nxt = ndist.pagerank_step(rp, ci, pr, od)
    torch.cuda.synchronize()
    want = opr.step(rp.cpu().numpy(), ci.cpu().numpy(), pr.cpu().numpy(), od.cpu().numpy())
    assert np.all(np.abs(nxt.cpu().numpy() - want) <= 1e-5 * want)


@pytest.mark.parametrize("P", [2, 3])
def test_fake_multigpu_pagerank_shards(cuda_device, P):
    # P node-row shards computed one after another on one GPU reassemble the full step
    from oracle import pagerank as opr
    from paper_conf_micro_leebsro14_b200 import npp
    from paper_conf_micro_leebsro14_b200.dist import shard_range
    N = 40000
    rp, ci, pr, od = gen.pagerank_inputs(N, avg_deg=12, seed=9, max_deg=800, device=cuda_device)
    parts = []
    for rank in range(P):
        lo, hi = shard_range(N, P, rank)
        e0, e1 = int(rp[lo]), int(rp[hi])
        parts.append(npp.pagerank_shard((rp[lo:hi + 1] - e0).contiguous(), ci[e0:e1].contiguous(), pr, od, lo, hi))
    torch.cuda.synchronize()
    want = opr.step(rp.cpu().numpy(), ci.cpu().numpy(), pr.cpu().numpy(), od.cpu().numpy())
    got = torch.cat(parts).cpu().numpy()
    assert np.all(np.abs(got - want) <= 1e-5 * want)

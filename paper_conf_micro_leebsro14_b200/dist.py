"""Multi-GPU partitioning of the nested patterns over torch.distributed (one process per GPU).

SURVEY.md §8e / DESIGN.md §8. The outer (storage-row) dimension of every input is split into contiguous
shards, one per rank. Where the rows are the Map level (sumRows, k-means points, logreg mini-batches)
the shards are independent problems and no collective runs (PageRank rows too, plus one all-gather
of the next vector per step). Where the rows are the level being
reduced (sumCols, the full-batch logreg gradient, the k-means centroid update) the shard results are a cross-device Split(P) of that
Reduce and NCCL adds them — the only data-path collective.

Every rank plans and executes its shard through libnpp.so (``compute=None``). The ``compute`` hook
exists so the host-side sharding and reduction logic can be tested on CPU with the gloo backend;
the product path never runs on the CPU.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(n: int, world: int, rank: int):
    """Contiguous, balanced shard [lo, hi) of n outer indices for `rank` (sizes differ by <= 1)."""
    base, extra = divmod(n, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


def _world(group):
    return dist.get_world_size(group), dist.get_rank(group)


def _npp():
    from . import npp  # raises if libnpp.so is missing: no CPU fallback
    return npp


def sum_rows(local: torch.Tensor, group=None, gather: bool = False, compute=None):
    """Row sums of this rank's row shard; rows are independent, so no collective unless `gather`."""
    out = compute(local) if compute is not None else _npp().sum_rows(local)
    if not gather:
        return out
    world, _ = _world(group)
    sizes = [torch.zeros(1, dtype=torch.int64, device=out.device) for _ in range(world)]
    dist.all_gather(sizes, torch.tensor([out.numel()], dtype=torch.int64, device=out.device), group=group)
    mx = int(max(int(s.item()) for s in sizes))
    buf = torch.zeros(mx, dtype=out.dtype, device=out.device)
    buf[: out.numel()] = out
    parts = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(parts, buf, group=group)
    return torch.cat([p[: int(s.item())] for p, s in zip(parts, sizes)])


def sum_cols(local: torch.Tensor, group=None, op: str = "all_reduce", dst: int = 0, compute=None):
    """Column sums of a row-sharded matrix: local column sums, then one NCCL reduction of [C]."""
    out = compute(local) if compute is not None else _npp().sum_cols(local)
    if op == "all_reduce":
        dist.all_reduce(out, op=dist.ReduceOp.SUM, group=group)
    elif op == "reduce":
        dist.reduce(out, dst=dst, op=dist.ReduceOp.SUM, group=group)
    else:
        raise ValueError(op)
    return out


def kmeans_assign(local_x: torch.Tensor, centroids: torch.Tensor, group=None, compute=None):
    """Assignments of this rank's points (centroids replicated); points are independent."""
    return compute(local_x, centroids) if compute is not None else _npp().kmeans_assign(local_x, centroids)


def kmeans_update(local_x: torch.Tensor, local_a: torch.Tensor, K: int, group=None, compute=None):
    """Per-centroid (Σ x, count) over all ranks' points: the local [K, D+1] partial of this rank's
    point shard, then one all-reduce of K*(D+1) floats (the groups are split across ranks: a
    cross-device Split of the groupBy's Reduce)."""
    u = compute(local_x, local_a, K) if compute is not None else _npp().kmeans_update(local_x, local_a, K)
    dist.all_reduce(u, op=dist.ReduceOp.SUM, group=group)
    return u


def pagerank_step(local_rowptr: torch.Tensor, local_colidx: torch.Tensor, pr: torch.Tensor, outdeg: torch.Tensor,
                  group=None, compute=None):
    """One PageRank step with the nodes (CSR rows) sharded: this rank's rows [lo, hi) of the in-neighbour
    CSR (local_rowptr rebased to 0, length hi-lo+1) against the replicated previous PageRank and
    out-degrees; the per-node contributions are computed over all N nodes, each rank writes its rows,
    and one all-gather assembles the next [N] vector (the exchange step of the iteration)."""
    N = pr.shape[0]
    world, rank = _world(group)
    lo, hi = shard_range(N, world, rank)
    if compute is not None:
        local = compute(local_rowptr, local_colidx, pr, outdeg, lo, hi)
    else:
        local = _npp().pagerank_shard(local_rowptr, local_colidx, pr, outdeg, lo, hi)
    parts = [torch.empty(b - a, dtype=local.dtype, device=local.device)
             for a, b in (shard_range(N, world, r) for r in range(world))]
    if all(p.numel() == parts[0].numel() for p in parts):
        dist.all_gather(parts, local, group=group)
    else:  # uneven shards: gather padded buffers
        mx = max(p.numel() for p in parts)
        buf = torch.zeros(mx, dtype=local.dtype, device=local.device)
        buf[: local.numel()] = local
        padded = [torch.empty(mx, dtype=local.dtype, device=local.device) for _ in range(world)]
        dist.all_gather(padded, buf, group=group)
        parts = [p[: q.numel()] for p, q in zip(padded, parts)]
    return torch.cat(parts)


def logreg_grad(local_x: torch.Tensor, local_y: torch.Tensor, w: torch.Tensor, batches: int, group=None,
                full_batch: bool = False, compute=None):
    """Per-mini-batch gradients of this rank's batches (independent), or with ``full_batch`` the
    gradient over all ranks' rows (local [1 x C] partial, then an all-reduce of C floats)."""
    fn = compute if compute is not None else _npp().logreg_grad
    g = fn(local_x, local_y, w, 1 if full_batch else batches)
    if full_batch:
        dist.all_reduce(g, op=dist.ReduceOp.SUM, group=group)
    return g

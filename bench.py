#!/usr/bin/env python
"""Benchmark of the nested-pattern hot path (BASELINE.json metric: achieved HBM GB/s for sumRows /
sumCols per shape, 1/2/4/8 GPU).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload paper|sumcols_1m4k|kmeans|logreg|rowscols]
                    [--strategy AUTO|LITERAL|1D|TB_T|WARP] [--impl reference] [--no-mappings]

A step (workload `paper`, the default) = sumRows and sumCols, AUTO mapping, at the paper's three shapes
[64K,1K], [8K,8K], [1K,64K] fp32 (Fig 3; BASELINE.json configs[1]) — six launches on six
distinct 256 MiB buffers, so every launch streams from HBM (inputs > L2, no flush needed).
At N > 1 each rank owns a row shard of [N*R, C] matrices (weak scaling): sumRows shards need no
exchange, sumCols partial column sums are all-reduced over NCCL (the one real exchange step).

Output: one JSON line on rank 0 (see DESIGN.md §9 for every key).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PAPER_SHAPES = [(65536, 1024), (8192, 8192), (1024, 65536)]
METRIC = "achieved HBM GB/s (% of B200 peak) for sumRows/sumCols per shape, 1/2/4/8 GPU"


def _fmt_shape(s):
    def k(v):
        return f"{v // 1048576}M" if v % 1048576 == 0 else (f"{v // 1024}K" if v % 1024 == 0 else str(v))
    return f"[{k(s[0])},{k(s[1])}]"


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs: torch copy, read+write)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic():
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    return json.load(open(p)) if os.path.exists(p) else {}


# ------------------------------------------------------------------------- clocks (NVML, sampled live)

class ClockSampler:
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, device_index: int, period_s: float = 0.0001):
        self.period = period_s
        self.samples, self.reasons = [], 0
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # noqa: BLE001
            self.err = str(e)
        self._stop = threading.Event()

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                self.reasons |= int(nv.nvmlDeviceGetCurrentClocksEventReasons(self.h))
            except Exception:  # noqa: BLE001
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self._t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "error": getattr(self, "err", "")}
        names = [n for bit, n in self.REASONS.items() if self.reasons & bit and n != "gpu_idle"]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": names, "samples": len(self.samples)}


# ------------------------------------------------------------------------- distributed plumbing

def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


# ------------------------------------------------------------------------- workloads

class Item:
    """One launch of the step: a plan, its device inputs/outputs, and its algorithmic bytes."""

    def __init__(self, name, plan, ins, out, algo_bytes):
        self.name, self.plan, self.ins, self.out, self.bytes = name, plan, ins, out, algo_bytes

    def run(self, stream, overlap=False):
        self.plan.execute(self.ins, self.out, stream=stream, overlap=overlap)


def build_paper(npp, gen, torch, rank, world, strategy, device):
    items, reduce_views = [], []
    col_total = sum(C for _, C in PAPER_SHAPES)
    col_buf = torch.empty(col_total, dtype=torch.float32, device=device)
    off = 0
    for si, (R, C) in enumerate(PAPER_SHAPES):
        for pattern in ("SUM_ROWS", "SUM_COLS"):
            seed = 300 + 2 * si + (pattern == "SUM_COLS")
            # rank r owns rows [r*R, (r+1)*R) of a [world*R, C] matrix (counter-based inputs)
            m = gen.uniform_f32(seed, (R, C), offset=rank * R * C, device=device)
            plan = npp.Plan(pattern, (R, C), "f32", strategy, device=device)
            if pattern == "SUM_COLS":
                out = col_buf[off:off + C]
                off += C
            else:
                out = plan.new_out()
            nbytes = R * C * 4 + out.numel() * 4
            items.append(Item(f"{pattern.lower()}{_fmt_shape((R, C))}", plan, [m], out, nbytes))
    if world > 1:
        reduce_views.append(col_buf)
    desc = "sumRows+sumCols fp32 @ [64K,1K],[8K,8K],[1K,64K] (paper shapes, Fig 3)"
    return items, reduce_views, desc


def build_sumcols_1m4k(npp, gen, torch, rank, world, strategy, device):
    R, C = 1 << 20, 4096
    r_local = R // world
    m = gen.uniform_f32(4, (r_local, C), offset=rank * r_local * C, device=device)
    plan = npp.Plan("SUM_COLS", (r_local, C), "f32", strategy, device=device)
    out = plan.new_out()
    items = [Item(f"sum_cols{_fmt_shape((r_local, C))}", plan, [m], out, r_local * C * 4 + C * 4)]
    return items, ([out] if world > 1 else []), "sumCols fp32 [1M,4K] row-sharded + NCCL all-reduce (strong)"


def build_kmeans(npp, gen, torch, rank, world, strategy, device):
    # BASELINE.json config 4: 4M points x 64 dims x 32 centroids; the points sharded over ranks (strong)
    Ntot, D, K = 1 << 22, 64, 32
    from paper_conf_micro_leebsro14_b200.dist import shard_range
    lo, hi = shard_range(Ntot, world, rank)
    N = hi - lo
    x, c = gen.kmeans_inputs(N, D, K, row_offset=lo, device=device)
    plan = npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", strategy, device=device)
    item = Item("kmeans_assign[4M,64,32]" if world == 1 else f"kmeans_assign[{N},64,32]", plan, [x, c],
                plan.new_out(), N * D * 4 + K * D * 4 + N * 4)
    item.flops = 2 * N * K * D  # the x·c FMAs of the expanded distance
    return [item], [], "k-means assignment 4M x 64 x 32"


def build_kmeans_update(npp, gen, torch, rank, world, strategy, device):
    # the centroid update after the config-4 assignment: 4M points x 64 dims into
    # 32 groups; keys = the generator's cluster labels of the same points (synthetic inputs, so the
    # cpu_baseline's oracle never consumes a CUDA result)
    N, D, K = 1 << 22, 64, 32
    x, c = gen.kmeans_inputs(N, D, K, row_offset=rank * N, device=device)
    a = gen.int_uniform(5 + 1, (N,), 0, K - 1, dtype=torch.int32, offset=rank * N, device=device)
    plan = npp.Plan("KMEANS_UPDATE", (N, D, K), "f32", "AUTO", device=device)
    out = plan.new_out()
    item = Item("kmeans_update[4M,64,32]", plan, [x, a], out, N * D * 4 + N * 4 + K * (D + 1) * 4)
    return [item], ([out] if world > 1 else []), "k-means centroid update 4M x 64 -> 32 groups"


def build_pagerank(npp, gen, torch, rank, world, strategy, device):
    # one PageRank step (Fig 5) over a 4M-node power-law graph (mean in-degree ~16,
    # cap 1024, ~63M edges). At N > 1 rank r computes its node rows [lo, hi) from its CSR shard against
    # the replicated previous vector, and the step ends with an all-gather of the next vector
    N = 1 << 22
    rowptr, colidx, pr, outdeg = gen.pagerank_inputs(N, avg_deg=16, seed=7, max_deg=1024, device=device)
    E = colidx.numel()
    if world == 1:
        plan = npp.Plan("PAGERANK", (N, E), "f32", "AUTO", device=device)
        item = Item("pagerank[4M,%dM]" % (E // 1000000), plan, [rowptr, colidx, pr, outdeg], plan.new_out(),
                    (N + 1) * 8 + E * 4 + N * 4 * 3)
        # the random gathers bound this path: one L1tex wavefront (128-B line) per edge for contrib[w], plus
        # the coalesced colidx / rowptr / per-node lines (DESIGN.md §6 PR)
        item.wavefronts = E + E * 4 // 128 + (N + 1) * 8 // 128 + 3 * N * 4 // 128
        return [item], [], "PageRank step, 4M nodes, ~63M edges"
    from paper_conf_micro_leebsro14_b200.dist import shard_range
    lo, hi = shard_range(N, world, rank)
    e0, e1 = int(rowptr[lo]), int(rowptr[hi])
    lrp = (rowptr[lo:hi + 1] - e0).contiguous()
    lci = colidx[e0:e1].contiguous()
    plan = npp.Plan("PAGERANK", (hi - lo, e1 - e0, N), "f32", "AUTO", device=device)
    item = Item("pagerank_shard[4M,%dM]" % (E // 1000000), plan, [lrp, lci, pr, outdeg], plan.new_out(),
                (hi - lo + 1) * 8 + (e1 - e0) * 4 + (hi - lo) * 4 + 2 * N * 4)
    item.gather = (world, N)
    return [item], [], "PageRank step, 4M nodes, ~63M edges, node rows sharded + all-gather"


def build_logreg(npp, gen, torch, rank, world, strategy, device):
    # BASELINE.json config 5: [16M, 256] fp32 in B = 4096 mini-batches of 4096 rows; batches sharded
    B, Rb, C = 4096 // world, 4096, 256
    x, y, w = gen.logreg_inputs(B, Rb, C, seed=6, batch_offset=rank * B, device=device)
    plan = npp.Plan("LOGREG_GRAD", (B, Rb, C), "f32", strategy, device=device)
    item = Item(f"logreg_grad[{B * Rb // 1048576}M,256]", plan, [x, y, w], plan.new_out(),
                B * Rb * C * 4 + B * Rb * 4 + C * 4 + B * C * 4)
    return [item], [], "batched logistic-regression gradient [16M,256], B=4096"


def build_rowscols(npp, gen, torch, rank, world, strategy, device):
    # the Naive Bayes counts (§VI-E): row AND column sums of each paper-shape matrix from
    # one pass (SUM_ROWS_COLS, S8 RC); rank r owns a row shard, the column sums are all-reduced
    items, col_views = [], []
    for si, (R, C) in enumerate(PAPER_SHAPES):
        m = gen.uniform_f32(300 + 2 * si, (R, C), offset=rank * R * C, device=device)
        plan = npp.Plan("SUM_ROWS_COLS", (R, C), "f32", "AUTO", device=device)
        out = plan.new_out()
        col_views.append(out[R:])
        items.append(Item(f"sum_rows_cols{_fmt_shape((R, C))}", plan, [m], out, R * C * 4 + (R + C) * 4))
    return items, (col_views if world > 1 else []), "sumRows and sumCols in one pass (Naive Bayes counts)"


# per-GPU work fixed as N grows ("weak": paper shards, k-means points) or total work fixed ("strong")
SCALING = {"paper": "weak", "kmeans": "strong", "sumcols_1m4k": "strong", "logreg": "strong", "rowscols": "weak",
           "kmeans_update": "weak", "pagerank": "strong"}
WORKLOADS = {"paper": build_paper, "sumcols_1m4k": build_sumcols_1m4k, "kmeans": build_kmeans,
             "logreg": build_logreg, "rowscols": build_rowscols, "kmeans_update": build_kmeans_update,
             "pagerank": build_pagerank}


# ------------------------------------------------------------------------- reference arm (the oracle)

def run_reference(args):
    """The reference arm: the oracle as it stands (NumPy fp64, one host core) on a bounded sample of
    the selected workload, same metric / unit / config as the npp arm."""
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    import numpy as np  # noqa: F401
    from oracle import kmeans as okm
    from oracle import logreg as olr
    from oracle import pagerank as opr
    from oracle import sums
    from synth import gen
    calls, desc = [], ""
    wl = args.workload
    if wl in ("paper", "sumcols_1m4k", "rowscols"):
        shapes = PAPER_SHAPES if wl != "sumcols_1m4k" else [(1 << 20, 4096)]
        sample_elems = 1 << 22   # the first rows of each matrix, 4M elements per (pattern, shape)
        for si, (R, C) in enumerate(shapes):
            rows = max(1, min(R, sample_elems // C))
            pats = {"paper": ("SUM_ROWS", "SUM_COLS"), "sumcols_1m4k": ("SUM_COLS",), "rowscols": ("SUM_ROWS_COLS",)}[wl]
            for pattern in pats:
                seed = (300 + 2 * si + (pattern == "SUM_COLS")) if wl != "sumcols_1m4k" else 4
                m = gen.uniform_f32(seed, (rows, C)).numpy()
                fn = {"SUM_ROWS": sums.sum_rows, "SUM_COLS": sums.sum_cols, "SUM_ROWS_COLS": sums.sum_rows_cols}[pattern]
                out = rows if pattern == "SUM_ROWS" else (C if pattern == "SUM_COLS" else rows + C)
                calls.append((lambda f=fn, a=m: f(a), m.size * 4 + out * 4))
        desc = f"first {sample_elems} elements of each matrix per step"
    elif wl in ("kmeans", "kmeans_update"):
        N, D, K = 1 << 16, 64, 32
        x, c = gen.kmeans_inputs(N, D, K)
        x, c = x.numpy(), c.numpy()
        if wl == "kmeans":
            calls.append((lambda: okm.assign(x, c), N * D * 4 + K * D * 4 + N * 4))
        else:
            a = okm.assign(x, c)
            calls.append((lambda: okm.update(x, a, K), N * D * 4 + N * 4 + K * (D + 1) * 4))
        desc = f"{N} points of the 4M x 64 x 32 workload per step"
    elif wl == "logreg":
        B, Rb, C = 16, 4096, 256
        x, y, w = gen.logreg_inputs(B, Rb, C, seed=6)
        x, y, w = x.numpy(), y.numpy(), w.numpy()
        calls.append((lambda: olr.grad(x, y, w, B), B * Rb * C * 4 + B * Rb * 4 + C * 4 + B * C * 4))
        desc = f"{B} of the 4096 mini-batches per step"
    elif wl == "pagerank":
        N = 1 << 20
        rp, ci, pr, od = (t.numpy() for t in gen.pagerank_inputs(N, avg_deg=16, seed=7, max_deg=1024))
        calls.append((lambda: opr.step(rp, ci, pr, od), (N + 1) * 8 + len(ci) * 4 + N * 12))
        desc = f"a {N}-node graph of the same recipe per step"
    step_bytes = sum(b for _, b in calls)

    def step():
        for f, _ in calls:
            f()
    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    dt = (time.perf_counter() - t0) / args.steps
    value = step_bytes / dt / 1e9
    line = {"metric": METRIC, "value": round(value, 3), "unit": "GB/s", "impl": "reference",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 3),
            "higher_is_better": True, "scaling": SCALING[wl], "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": config_for(args, "oracle (NumPy fp64) on host cores"),
            "cpu_baseline": {"value": round(value, 3), "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": desc, "cpu_model": _cpu_model(), "cpu_count": os.cpu_count()},
            "e2e": {"value": round(value, 3), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def config_for(args, extra):
    wl = {"paper": "sumRows+sumCols fp32 @ [64K,1K],[8K,8K],[1K,64K] (paper shapes, BASELINE.json configs[1])",
          "sumcols_1m4k": "sumCols fp32 [1M,4K] row-sharded (BASELINE.json configs[2])",
          "kmeans": "k-means assignment 4M x 64 x 32 fp32, points sharded (BASELINE.json configs[3])",
          "logreg": "batched logreg gradient [16M,256] fp32, B=4096, batches sharded (BASELINE.json configs[4])",
          "pagerank": "PageRank step (Fig 5) over a 4M-node power-law CSR graph, ~63M edges fp32 (SURVEY §8f "
                      "NEXT 4)",
          "kmeans_update": "k-means centroid update 4M x 64 -> 32 groups fp32, points sharded + all-reduce "
                           "of [32, 65] (SURVEY §8f NEXT 4)",
          "rowscols": "sumRows+sumCols in ONE pass (SUM_ROWS_COLS) fp32 @ [64K,1K],[8K,8K],[1K,64K] "
                      "(Naive Bayes counts, SURVEY §8f NEXT 2)",
          }[args.workload]
    return {"workload": wl, "strategy": args.strategy, "impl_detail": extra,
            "parallelism": f"row shards x{args.gpus}",
            "l2": "inputs larger than L2 (distinct 256 MiB buffers per launch, 1.5 GiB per step); no flush"}


# ------------------------------------------------------------------------- CPU baseline (oracle, bounded)

def _oracle_call(name, arrs, k=0):
    from oracle import kmeans as okm
    from oracle import logreg as olr
    from oracle import pagerank as opr
    from oracle import sums
    if name.startswith("pagerank"):
        opr.step(*arrs)
    elif name.startswith("kmeans_update"):
        okm.update(arrs[0], arrs[1], k)
    elif name.startswith("kmeans"):
        okm.assign(*arrs)
    elif name.startswith("logreg"):
        olr.grad(arrs[0], arrs[1], arrs[2], arrs[0].shape[0] // 4096)
    elif name.startswith("sum_rows_cols"):
        sums.sum_rows_cols(arrs[0])
    elif name.startswith("sum_rows"):
        sums.sum_rows(arrs[0])
    else:
        sums.sum_cols(arrs[0])


def _pool_worker(job):
    """One process of the all-core CPU baseline: run the oracle on its slice of the sample."""
    import numpy as np  # noqa: F401
    name, arrs, k, reps = job
    t0 = time.perf_counter()
    for _ in range(reps):
        _oracle_call(name, arrs, k)
    return time.perf_counter() - t0


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_baseline(items, budget_s=10.0):
    """The oracle as it stands (NumPy fp64) on a bounded sample of the same workload, timed on one
    core and as a process pool over all cores, plus the literal (pure-Python) oracle
    on [1K,1K]."""
    import multiprocessing as mp

    import numpy as np
    from oracle import sums
    samples = []
    k = 0
    for it in items:
        if it.name.startswith("pagerank"):  # the whole graph (the oracle is O(E) NumPy)
            samples.append((it.name, [x.cpu().numpy() for x in it.ins]))
        elif it.name.startswith("kmeans_update"):  # first 1M points
            k = it.plan.shape[2]
            samples.append((it.name, [it.ins[0][: 1 << 20].cpu().numpy(), it.ins[1][: 1 << 20].cpu().numpy()]))
        elif it.name.startswith("kmeans"):  # first 128K points (the oracle is O(N K D) in fp64)
            samples.append((it.name, [it.ins[0][: 1 << 17].cpu().numpy(), it.ins[1].cpu().numpy()]))
        elif it.name.startswith("logreg"):  # first 16 batches
            rows = 16 * it.plan.shape[1]
            samples.append((it.name, [it.ins[0][:rows].cpu().numpy(), it.ins[1][:rows].cpu().numpy(),
                                      it.ins[2].cpu().numpy()]))
        else:  # the first 16 MB of each matrix
            m = it.ins[0]
            rows = max(1, min(m.shape[0], (1 << 22) // m.shape[1]))
            samples.append((it.name, [m[:rows].cpu().numpy()]))
    sample_bytes = sum(x.nbytes for _, arrs in samples for x in arrs)
    # one core: passes over the sample until the budget is spent
    t_total, n_pass = 0.0, 0
    t_end = time.perf_counter() + budget_s / 2
    while time.perf_counter() < t_end:
        for name, arrs in samples:
            t0 = time.perf_counter()
            _oracle_call(name, arrs, k)
            t_total += time.perf_counter() - t0
        n_pass += 1
    one_core = sample_bytes * n_pass / t_total / 1e9
    # all cores: one process per core, each running the oracle over the sample (independent work)
    try:
        cores = len(os.sched_getaffinity(0))  # the cores this process may run on (os.cpu_count() counts all)
    except AttributeError:
        cores = os.cpu_count() or 1
    reps = max(1, n_pass // 2)
    jobs = [(name, arrs, k, reps) for name, arrs in samples for _ in range(cores)]
    try:
        ctx = mp.get_context("fork")
        t0 = time.perf_counter()
        with ctx.Pool(cores) as pool:
            pool.map(_pool_worker, jobs, chunksize=1)
        wall = time.perf_counter() - t0
        all_core = sample_bytes * reps * cores / wall / 1e9
    except Exception as e:  # noqa: BLE001
        all_core, wall = None, str(e)
    # the literal oracle (pure-Python loops) on [1K,1K] fp32
    m = np.random.default_rng(1).random((1024, 1024), dtype=np.float32)
    t0 = time.perf_counter()
    sums.sum_rows_literal(m)
    sums.sum_cols_literal(m)
    literal_s = time.perf_counter() - t0
    return {"value": round(all_core if all_core else one_core, 3), "unit": "GB/s",
            "cores": cores if all_core else 1, "kind": "oracle",
            "one_core_GBps": round(one_core, 3), "all_core_GBps": round(all_core, 3) if all_core else None,
            "cpu_model": _cpu_model(), "cpu_count": os.cpu_count(),
            "literal_1k_rows_cols_s": round(literal_s, 3),
            "sample": f"{len(samples)} oracle calls per pass over the first 16 MB of each matrix (k-means: "
                      f"first 128K points, logreg: first 16 batches); one core: {n_pass} passes "
                      f"({t_total:.1f} s); all cores: {cores} processes x {reps} passes "
                      f"({wall if isinstance(wall, str) else round(wall, 1)} s); NumPy fp64"}


# ------------------------------------------------------------------------- timing plumbing

def torchrun_cmd(gpus: int, port: int, argv) -> list:
    """The command that runs this bench as `gpus` ranks of one node (rendezvous on 127.0.0.1)."""
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={gpus}",
            "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + list(argv)


def self_launch(args) -> int:
    """`python bench.py --gpus N` outside torchrun: re-run this command as N ranks (one per GPU)."""
    import socket
    import subprocess
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return subprocess.call(torchrun_cmd(args.gpus, port, sys.argv[1:]))


def capture_step(torch, step, stream, world):
    """The step as a CUDA graph (kernels and, at N > 1, the NCCL collectives): the timed region replays
    it, so every N times the same way. Returns (replay, how)."""
    with torch.cuda.stream(stream):
        step()  # warm: lazy per-kernel setup, NCCL communicator, tensor maps
    torch.cuda.synchronize()
    try:
        g = torch.cuda.CUDAGraph()
        with torch.cuda.stream(stream):
            with torch.cuda.graph(g, stream=stream):
                step()
        torch.cuda.synchronize()
        return g.replay, "CUDA graph" + (" (kernels + NCCL)" if world > 1 else "")
    except Exception as e:  # noqa: BLE001  (a capture failure must not lose the measurement)
        torch.cuda.synchronize()
        return step, f"eager launches (graph capture failed: {type(e).__name__})"


def timed(torch, dist, run_step, stream, steps, world, local):
    """Barrier + sync, CUDA events on `stream` around `steps` replays, clocks sampled live; the max over
    ranks. Returns (ms_total_max, per_rank_ms, clocks)."""
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(local)
    with sampler:
        with torch.cuda.stream(stream):
            t0.record(stream)
            for _ in range(steps):
                run_step()
            t1.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = t0.elapsed_time(t1)
    per_rank = [ms]
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=torch.device("cuda", local))
        parts = [torch.zeros_like(t) for _ in range(world)]
        dist.all_gather(parts, t)
        per_rank = [float(x.item()) for x in parts]
    return max(per_rank), per_rank, sampler.summary()


def kernel_us(torch, item, other, stream, reps=8, overlap=False, pdl=False):
    """Average duration of one launch of item's plan: a graph of 2*reps launches alternating item's
    input with `other`'s (same byte size) so no launch finds its input in L2. Default: plain launches
    (NPP_EXEC_NO_PDL: each kernel starts after the previous one completed — the isolated duration the
    roofline uses); pdl=True: programmatic dependent launches (prologue overlapped, reads still after the
    previous kernel); overlap=True: NPP_EXEC_OVERLAP (reads overlap the previous kernel's drain)."""
    alt = None
    if other is not None and other.ins[0].numel() == item.ins[0].numel() and other.ins[0].dtype == item.ins[0].dtype:
        alt = other.ins[0].view(item.ins[0].shape)
    firsts = [item.ins[0], alt] if alt is not None and alt.data_ptr() != item.ins[0].data_ptr() else [item.ins[0]]
    inputs = [[f] + list(item.ins[1:]) for f in firsts]
    use_pdl = pdl or overlap
    with torch.cuda.stream(stream):
        for x in inputs:
            item.plan.execute(x, item.out, stream=stream, pdl=use_pdl)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(stream):
        with torch.cuda.graph(g, stream=stream):
            for r in range(2 * reps):
                item.plan.execute(inputs[r % len(inputs)], item.out, stream=stream, overlap=overlap, pdl=use_pdl)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        g.replay()
        a.record(stream)
        g.replay()
        b.record(stream)
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1e3 / (2 * reps)


def make_step(torch, dist, items, reduce_bufs, stream, world, overlap):
    gathers = [it for it in items if getattr(it, "gather", None)]

    def step():
        for it in items:
            it.run(stream, overlap)
        for b in reduce_bufs:  # the cross-device Split(P) of a reduced level: one NCCL all-reduce
            with torch.cuda.stream(stream):
                dist.all_reduce(b)
        for it in gathers:  # PageRank shards: the next vector on every rank (uneven shards padded)
            with torch.cuda.stream(stream):
                n = it.out.numel()
                mx = -(-it.gather[1] // world)
                buf = torch.zeros(mx, dtype=it.out.dtype, device=it.out.device)
                buf[:n] = it.out
                parts = [torch.empty(mx, dtype=it.out.dtype, device=it.out.device) for _ in range(world)]
                dist.all_gather(parts, buf)
    return step


# ------------------------------------------------------------------------- main arm

def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="paper", choices=sorted(WORKLOADS))
    ap.add_argument("--strategy", default="AUTO")
    ap.add_argument("--impl", default="npp", choices=["npp", "reference"])
    ap.add_argument("--no-mappings", action="store_true", help="skip the baseline-mapping table")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-e2e", action="store_true", help="skip the host-buffer e2e leg")
    ap.add_argument("--no-per-config", action="store_true", help="skip the per_config lines (configs 3-5)")
    ap.add_argument("--eager", action="store_true", help="time eager launches instead of a CUDA graph")
    ap.add_argument("--no-overlap", action="store_true",
                    help="serialise the step's launches (no NPP_EXEC_OVERLAP programmatic dependent launch)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return self_launch(args)

    import torch
    import torch.distributed as dist
    from paper_conf_micro_leebsro14_b200 import npp
    from synth import gen

    world, rank, local = dist_env()
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    device = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=device)
    items, reduce_bufs, _ = WORKLOADS[args.workload](npp, gen, torch, rank, world, args.strategy, device)
    stream = torch.cuda.Stream(device=device)  # all timed work is enqueued on this stream

    # the step's inputs are resident before it starts, so each launch may overlap the previous one's
    # drain (npp_execute_ex NPP_EXEC_OVERLAP); outputs still wait for the previous kernel
    overlap = not args.no_overlap
    step = make_step(torch, dist, items, reduce_bufs, stream, world, overlap)
    if args.eager:
        with torch.cuda.stream(stream):
            step()
        run_step, how = step, "eager launches"
    else:
        run_step, how = capture_step(torch, step, stream, world)
    with torch.cuda.stream(stream):
        for _ in range(max(3, args.warmup)):
            run_step()
    ms_total, per_rank_ms, clocks = timed(torch, dist, run_step, stream, args.steps, world, local)
    ms_step = ms_total / args.steps
    step_bytes = sum(it.bytes for it in items)
    value = step_bytes * world / (ms_step * 1e-3) / 1e9

    # per-kernel durations: each launch replayed back to back from a graph, alternating its input with
    # another equal-size buffer of the step so that every launch reads cold HBM
    nxt = [items[(i + 1) % len(items)] if len(items) > 1 else None for i in range(len(items))]
    per_kernel_us = [kernel_us(torch, it, nxt[i], stream) for i, it in enumerate(items)]
    per_kernel_pdl = [kernel_us(torch, it, nxt[i], stream, pdl=True) for i, it in enumerate(items)]
    per_kernel_ov = [kernel_us(torch, it, nxt[i], stream, overlap=True) for i, it in enumerate(items)]
    peak, peak_src = measured_peaks()
    dom = max(range(len(items)), key=lambda i: per_kernel_us[i])
    traffic_db = ncu_traffic()

    def gbps(it, us):
        return it.bytes / (us * 1e-6) / 1e9
    per_shape = {}
    for i, it in enumerate(items):
        ent = {"GB/s": round(gbps(it, per_kernel_us[i]), 1), "us": round(per_kernel_us[i], 2),
               "frac_of_measured": round(gbps(it, per_kernel_us[i]) / peak, 4),
               "frac_of_8TBs": round(gbps(it, per_kernel_us[i]) / 8000.0, 4),
               "us_pdl": round(per_kernel_pdl[i], 2), "us_overlapped": round(per_kernel_ov[i], 2),
               "GB/s_overlapped": round(gbps(it, per_kernel_ov[i]), 1), "mapping": mapping_brief(it.plan.mapping)}
        ncu_us = traffic_db.get(it.name + "/ncu_us")
        if ncu_us:  # ncu-isolated duration (cold cache, serialised; profiles/ncu_traffic.json)
            ent["ncu_us"] = ncu_us
            ent["ncu_GBps"] = round(gbps(it, ncu_us), 1)
            ent["ncu_dram_GBps"] = round(traffic_db.get(it.name, 0) / (ncu_us * 1e-6) / 1e9, 1)
        per_shape[it.name] = ent

    out = {"metric": METRIC, "value": round(value, 1), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(ms_step, 4), "higher_is_better": True,
           "scaling": SCALING[args.workload], "vs_baseline": None, "dtype": "f32",
           "data": "synthetic (counter-based U[0,1) fp32, seeded)",
           "config": dict(config_for(args, f"libnpp.so sm_100a; step replayed as {how}"),
                          launches="programmatic dependent launch (NPP_EXEC_OVERLAP)" if overlap
                          else "serialised", timing="CUDA events on the launching stream, max over ranks"),
           "gpu_launches": args.steps * sum(it.plan.launches for it in items),
           "per_rank_GBps": [round(step_bytes / (ms / args.steps * 1e-3) / 1e9, 1) for ms in per_rank_ms],
           "clocks": clocks,
           "roofline": roofline(items[dom], per_kernel_us[dom], gbps(items[dom], per_kernel_us[dom]), peak,
                                peak_src, traffic_db.get(items[dom].name), getattr(items[dom], "flops", None),
                                getattr(items[dom], "wavefronts", None)),
           "per_shape": per_shape}

    # e2e: same metric through the C-ABI with HOST buffers (H2D of the inputs + D2H of the result inside)
    out["e2e"] = None if args.no_e2e else e2e_host(items, torch, stream, world, dist)
    if rank == 0 and not args.no_mappings and args.workload == "paper":
        out["mappings"] = mapping_table(npp, torch, device, stream, items)
        out["fused_rows_cols"] = fused_table(npp, torch, device, stream, items, per_shape)
    if rank == 0 and world == 1 and not args.no_cpu:
        out["cpu_baseline"] = cpu_baseline(items)
    if not args.no_per_config and args.workload == "paper":
        del items, step, run_step
        torch.cuda.empty_cache()
        out["per_config"] = per_config(npp, gen, torch, dist, world, rank, local, device, args, peak, peak_src)
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


PER_CONFIG = [("sumcols_1m4k", "BASELINE.json configs[2]: sumCols [1M,4K] fp32, rows sharded + NCCL all-reduce"),
              ("kmeans", "configs[3]: k-means assignment 4M x 64 x 32, points sharded"),
              ("logreg", "configs[4]: logreg gradient [16M,256] fp32, B=4096, batches sharded")]


def per_config(npp, gen, torch, dist, world, rank, local, device, args, peak, peak_src):
    """BASELINE.json configs 3-5 at this run's N (strong scaling: the config's total work split over the
    ranks), each timed like the step (graph replay, CUDA events, max over ranks, clocks sampled live in
    a timed region of >= 25 ms) with the roofline of its kernel (isolated launches)."""
    res = {}
    stream = torch.cuda.Stream(device=device)
    for wl, desc in PER_CONFIG:
        items, reduce_bufs, _ = WORKLOADS[wl](npp, gen, torch, rank, world, "AUTO", device)
        step = make_step(torch, dist, items, reduce_bufs, stream, world, True)
        run_step, how = capture_step(torch, step, stream, world)
        with torch.cuda.stream(stream):
            for _ in range(3):
                run_step()
        ms_probe, _, _ = timed(torch, dist, run_step, stream, 2, world, local)
        steps = max(args.steps, int(math.ceil(25.0 / max(ms_probe / 2, 1e-3))))
        ms_total, per_rank_ms, clocks = timed(torch, dist, run_step, stream, steps, world, local)
        ms_step = ms_total / steps
        step_bytes = sum(it.bytes for it in items)
        it = items[0]
        us = kernel_us(torch, it, None, stream, reps=4)
        rl = roofline(it, us, it.bytes / (us * 1e-6) / 1e9, peak, peak_src, ncu_traffic().get(it.name),
                      getattr(it, "flops", None))
        res[wl] = {"value": round(step_bytes * world / (ms_step * 1e-3) / 1e9, 1), "unit": "GB/s",
                   "ms_per_step": round(ms_step, 4), "steps": steps, "scaling": SCALING[wl], "timing": how,
                   "per_rank_GBps": [round(step_bytes / (ms / steps * 1e-3) / 1e9, 1) for ms in per_rank_ms],
                   "roofline": {k: rl[k] for k in ("kernel", "bound", "achieved", "peak", "unit", "frac",
                                                   "duration_us", "hbm_GBps", "traffic")},
                   "clocks": clocks, "config": desc}
        del items, step, run_step, reduce_bufs
        torch.cuda.empty_cache()
        if world > 1 and wl == "sumcols_1m4k":
            # strong scaling of config 3: the whole [1M,4K] on rank 0 alone (the other ranks wait at the
            # barrier), the same graph-timed way, against this run's N-rank time
            t1_ms = None
            if rank == 0:
                items1, _, _ = WORKLOADS[wl](npp, gen, torch, 0, 1, "AUTO", device)
                step1 = make_step(torch, dist, items1, [], stream, 1, True)
                run1, _ = capture_step(torch, step1, stream, 1)
                with torch.cuda.stream(stream):
                    for _ in range(3):
                        run1()
                t1_total, _, _ = timed(torch, dist, run1, stream, steps, 1, local)
                t1_ms = t1_total / steps
                del items1, step1, run1
                torch.cuda.empty_cache()
            dist.barrier()
            if rank == 0:
                res[wl]["T1_ms"] = round(t1_ms, 4)
                res[wl]["T1_over_P_TP"] = round(t1_ms / (world * ms_step), 4)
    return res


def roofline(item, us, gbs, peak, peak_src, traffic, flops, wavefronts=None):
    base = {"kernel": item.name, "traffic": traffic, "algorithmic_bytes": item.bytes, "duration_us": round(us, 2),
            "hbm_GBps": round(gbs, 1), "hbm_frac_of_measured": round(gbs / peak, 4),
            "timing": "isolated launches (NPP_EXEC_NO_PDL), L2-cold, CUDA events"}
    if wavefronts:  # random gathers: L1tex wavefront rate, ~1 per cycle per SM (B300_MICROARCH.md LDG model)
        wf_peak = 148 * 1.965e9 / 1e9
        achieved = wavefronts / (us * 1e-6) / 1e9
        return dict(base, bound="l1tex", achieved=round(achieved, 2), peak=round(wf_peak, 2),
                    unit="G wavefronts/s", frac=round(achieved / wf_peak, 4),
                    peak_source="derived: 148 SM x 1 L1tex wavefront/clk (guide: rt_L1tex_wf ~ 1.0 cyc/wf) x 1965 MHz",
                    algorithmic_wavefronts=wavefronts)
    if flops:  # FP32 FMA-bound (k-means): peak = 148 SMs x 128 FP32 lanes x 2 flop x 1965 MHz
        alu_peak = 148 * 128 * 2 * 1.965e9 / 1e12
        achieved = flops / (us * 1e-6) / 1e12
        return dict(base, bound="alu", achieved=round(achieved, 2), peak=round(alu_peak, 2), unit="TFLOP/s",
                    frac=round(achieved / alu_peak, 4),
                    peak_source="derived: 148 SM x 128 FP32 FMA/clk x 2 x 1965 MHz (guide unit counts)",
                    algorithmic_flops=flops,
                    # measured context (profiles/r02/kmeans/micro_inner.log): the kernel's dims loop alone, with
                    # its 4-point x 8-centroid thread tile, reaches 0.63-0.69 of this peak — one uniform
                    # constant-bank load per 4 packed FMAs, not the FMA pipe, sets that ceiling
                    dims_loop_alone_frac=[0.63, 0.69])
    return dict(base, bound="hbm", achieved=round(gbs, 1), peak=peak, peak_source=peak_src, unit="GB/s",
                frac=round(gbs / peak, 4))


def mapping_brief(m):
    def span(l):
        return {0: "Span(1)", 1: "Span(all)", 2: f"Span({l['factor']})", 3: f"Split({l['factor']})"}[l["span"]]
    dims = "xyz"
    return "; ".join(f"L{i}:{dims[l['dim']]},{l['block']},{span(l)}" for i, l in enumerate(m["levels"])) + \
        f"; vec={m['vec']}; grid={m['grid']}"


def e2e_host(items, torch, stream, world, dist, steps=3):
    host_ins = [[x.cpu().pin_memory() for x in it.ins] for it in items]
    host_outs = [torch.empty(it.out.shape, dtype=it.out.dtype).pin_memory() for it in items]
    h2d = sum(h.numel() * h.element_size() for hs in host_ins for h in hs)
    d2h = sum(h.numel() * h.element_size() for h in host_outs)

    def one():
        for it, hi, ho in zip(items, host_ins, host_outs):
            it.plan.execute_host(hi, ho, it.ins, it.out, stream=stream)
    one()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(steps):
        one()
    dt = (time.perf_counter() - t0) / steps
    if world > 1:
        t = torch.tensor([dt], dtype=torch.float64, device=items[0].out.device)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dt = float(t.item())
    value = sum(it.bytes for it in items) * world / dt / 1e9
    return {"value": round(value, 2), "unit": "GB/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "steps": steps, "api": "npp_execute_host (pinned host buffers, blocking)"}


def fused_table(npp, torch, device, stream, items, per_shape):
    """Both sums of one matrix: the one-pass SUM_ROWS_COLS launch vs the sumRows + sumCols launches
    (isolated, L2-cold like per_shape). GB/s counts the one algorithmic read + both outputs."""
    table = {}
    flat = [it.ins[0] for it in items]
    for R, C in PAPER_SHAPES:
        m = next(x for x in flat if tuple(x.shape) == (R, C))
        other = next(x for x in flat if x.data_ptr() != m.data_ptr() and x.numel() == m.numel())
        p = npp.Plan("SUM_ROWS_COLS", (R, C), "f32", "AUTO", device=device)
        item = Item("rc", p, [m], p.new_out(), R * C * 4 + (R + C) * 4)
        us = kernel_us(torch, item, Item("o", p, [other], None, 0), stream)
        two = per_shape[f"sum_rows{_fmt_shape((R, C))}"]["us"] + per_shape[f"sum_cols{_fmt_shape((R, C))}"]["us"]
        table[f"sum_rows_cols{_fmt_shape((R, C))}"] = {
            "GB/s": round(item.bytes / (us * 1e-6) / 1e9, 1), "us": round(us, 2), "two_pass_us": round(two, 2),
            "speedup": round(two / us, 3)}
    return table


def mapping_table(npp, torch, device, stream, items):
    """The paper's Fig 3 comparison on B200: GB/s of every strategy at every paper shape (isolated
    launches, L2-cold)."""
    table = {}
    bufs = {}
    for it in items:
        bufs.setdefault(tuple(it.ins[0].shape), []).append(it.ins[0])
    flat = [it.ins[0] for it in items]
    for R, C in PAPER_SHAPES:
        m = bufs[(R, C)][0]
        other = next(x for x in flat if x.data_ptr() != m.data_ptr() and x.numel() == m.numel())
        for pattern in ("SUM_ROWS", "SUM_COLS"):
            row = {}
            for strat in ("AUTO", "LITERAL", "1D", "TB_T", "WARP"):
                p = npp.Plan(pattern, (R, C), "f32", strat, device=device)
                item = Item(pattern, p, [m], p.new_out(), R * C * 4)
                reps = 8 if strat in ("AUTO", "LITERAL", "WARP") else 2
                us = kernel_us(torch, item, Item("o", p, [other], None, 0), stream, reps=reps)
                row[strat] = round((R * C * 4 + item.out.numel() * 4) / (us * 1e-6) / 1e9, 1)
            table[f"{pattern.lower()}{_fmt_shape((R, C))}"] = row
    return table


if __name__ == "__main__":
    sys.exit(main())

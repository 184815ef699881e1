"""One small invocation of every kernel family of libnpp.so, for compute-sanitizer
(memcheck / racecheck / synccheck):

    compute-sanitizer --tool memcheck --error-exitcode 1 python tools/sanitize_run.py

Covers: staged sums (narrow/wide tiles, RX/MX, f32/i32/i64, ragged edges, pool + combiner, PDL
overlap), weighted staged sums, the direct-load family under every strategy (Split(k) combine), the
S10 temp family (PREALLOC layouts and MALLOC), k-means assignment, logreg gradient, the one-pass
rows+cols family (staged and direct, regions cut both ways), the k-means update, the PageRank step
(full graph and a shard).
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_micro_leebsro14_b200 import npp  # noqa: E402
from synth import gen  # noqa: E402


def main():
    dev = torch.device("cuda:0")
    n = 0
    for dtype in ("f32", "i32", "i64"):
        for shape in [(300, 1024), (67, 520), (1000, 36), (5, 3)]:
            m = (gen.uniform_f32(1, shape, device=dev) if dtype == "f32" else
                 gen.int_uniform(2, shape, -50, 50, device=dev) if dtype == "i32" else
                 gen.int64_wide(3, shape, device=dev))
            for pattern in ("SUM_ROWS", "SUM_COLS"):
                for strat in ("AUTO", "LITERAL", "1D", "TB_T", "WARP"):
                    p = npp.Plan(pattern, shape, dtype, strat)
                    p.execute([m], p.new_out())
                    p.execute([m], p.new_out(), overlap=True)
                    n += 2
            for pattern, vlen in (("SUM_WEIGHTED_ROWS", shape[1]), ("SUM_WEIGHTED_COLS", shape[0])):
                v = m[0, :vlen].contiguous() if pattern == "SUM_WEIGHTED_ROWS" else m[:vlen, 0].contiguous()
                for strat in ("AUTO", "LITERAL"):
                    p = npp.Plan(pattern, shape, dtype, strat)
                    p.execute([m, v], p.new_out())
                    n += 1
                if dtype != "i64":
                    lit = npp.Plan(pattern, shape, dtype, "LITERAL").mapping
                    M, N = (shape[0], shape[1]) if pattern == "SUM_WEIGHTED_ROWS" else (shape[1], shape[0])
                    for rec in (dict(lit, temp_stride=[N, 1]), dict(lit, temp=npp.TEMP_MALLOC, temp_stride=[0, 1])):
                        p = npp.Plan(pattern, shape, dtype, mapping=rec)
                        p.execute([m, v], p.new_out())
                        n += 1
    x, c = gen.kmeans_inputs(5000, 64, 32, device=dev)
    npp.Plan("KMEANS_ASSIGN", (5000, 64, 32)).execute([x, c], torch.empty(5000, dtype=torch.int32, device=dev))
    x, c = gen.kmeans_inputs(700, 96, 40, device=dev)
    npp.Plan("KMEANS_ASSIGN", (700, 96, 40)).execute([x, c], torch.empty(700, dtype=torch.int32, device=dev))
    # near ties: exact midpoints of centroid pairs run the fp64 recheck path (D = 64 and D = 32 kernels)
    for D in (64, 32):
        cc = (torch.randint(-64, 64, (32, D), generator=torch.Generator().manual_seed(D)).float() / 4.0).to(dev)
        xx = ((cc[torch.arange(600) % 32] + cc[(torch.arange(600) * 7 + 3) % 32]) / 2).contiguous()
        npp.Plan("KMEANS_ASSIGN", (600, D, 32)).execute([xx, cc], torch.empty(600, dtype=torch.int32, device=dev))
        n += 1
    # traced schedules and plain (non-PDL) launches
    mt = gen.uniform_f32(7, (4097, 300), device=dev)
    for pattern in ("SUM_ROWS", "SUM_COLS", "SUM_ROWS_COLS"):
        p = npp.Plan(pattern, (4097, 300), "f32", "AUTO")
        p.execute_traced([mt], p.new_out())
        p.execute([mt], p.new_out(), pdl=False)
        n += 2
    lx, ly, lw = gen.logreg_inputs(5, 100, 256, device=dev)
    npp.Plan("LOGREG_GRAD", (5, 100, 256)).execute([lx, ly, lw], torch.empty(5, 256, device=dev))
    n += 3
    for dtype in ("f32", "i32", "i64"):
        for shape in [(300, 1024), (1000, 999), (64, 9000), (5, 3)]:
            m = (gen.uniform_f32(4, shape, device=dev) if dtype == "f32" else
                 gen.int_uniform(5, shape, -50, 50, device=dev) if dtype == "i32" else
                 gen.int64_wide(6, shape, device=dev))
            p = npp.Plan("SUM_ROWS_COLS", shape, dtype)
            p.execute([m], p.new_out())
            p.execute([m], p.new_out(), overlap=True)
            n += 2
    for N, D, K in [(3000, 64, 32), (517, 8, 100), (129, 4, 1)]:
        x, _ = gen.kmeans_inputs(N, D, K, device=dev)
        a = gen.int_uniform(7, (N,), -1, K, device=dev)
        p = npp.Plan("KMEANS_UPDATE", (N, D, K))
        p.execute([x, a], p.new_out())
        p.execute([x, a], p.new_out(), overlap=True)
        n += 2
    rp, ci, pr, od = gen.pagerank_inputs(3000, avg_deg=10, seed=2, max_deg=400, device=dev)
    npp.pagerank_step(rp, ci, pr, od)
    lo, hi = 1000, 2500
    npp.pagerank_shard((rp[lo:hi + 1] - rp[lo]).contiguous(), ci[int(rp[lo]):int(rp[hi])].contiguous(), pr, od, lo, hi)
    n += 2
    torch.cuda.synchronize()
    print(f"sanitize_run ok: {n} executes")


if __name__ == "__main__":
    main()

"""Score-vs-performance sweep over the mapping space (§VI-G, Fig 17) on B200.

For sumRows and sumCols at the paper's three shapes, every hard-feasible Algorithm 1 candidate
(npp_enumerate: S2-S6, ControlDOP applied, recorded as LITERAL) is executed through
npp_plan_with_mapping on the direct-load kernel family and timed; AUTO (R2 + staged TMA family),
LITERAL (the selector's pick), TB/T, warp-based and 1D are timed as markers.

    python tools/sweep_fig17.py [--out gpurun_out/fig17.json] [--shapes 65536x1024,...]
    python tools/sweep_fig17.py --summarize gpurun_out/fig17.json    # markdown summary (no GPU)

Timing: CUDA events around a graph of launches alternating two distinct 256 MiB inputs (L2-cold),
median of 3 replays; algorithmic bytes = R*C*4 + outputs*4. Every mapping is first executed once and its
output checked against the oracle (|out - oracle| <= 1e-5 * Σ|terms|); a mapping that fails is recorded
with "valid": false and not timed.
"""
from __future__ import annotations

import argparse
import json
import re

import numpy as np
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SHAPES = [(65536, 1024), (8192, 8192), (1024, 65536), (50, 20000)]  # + the paper's skewed shape (L1362-1363)
SPAN = {0: "1", 1: "all", 2: "n", 3: "split"}


def brief(m):
    out = []
    for l in m["levels"]:
        sp = SPAN[l["span"]]
        if sp in ("n", "split"):
            sp = f"{sp}({l['factor']})"
        out.append(f"{'xyz'[l['dim']]}{l['block']}/{sp}")
    return " ".join(out)


def time_plan(torch, plan, ins_a, ins_b, out, stream, budget_ms=400.0, slow_ms=20.0):
    """Median per-launch microseconds of a graph alternating two inputs."""
    with torch.cuda.stream(stream):
        plan.execute(ins_a, out, stream=stream)
        plan.execute(ins_b, out, stream=stream)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    with torch.cuda.stream(stream):
        plan.execute(ins_a, out, stream=stream)
    torch.cuda.synchronize()
    one_ms = (time.perf_counter() - t0) * 1e3
    if one_ms > slow_ms:  # a very slow mapping: one more event-timed launch is precise enough
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            a.record(stream)
            plan.execute(ins_b, out, stream=stream)
            b.record(stream)
        torch.cuda.synchronize()
        return a.elapsed_time(b) * 1e3
    n = int(max(2, min(16, budget_ms / max(one_ms, 1e-3) / 3)))
    n += n % 2
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(stream):
        with torch.cuda.graph(g, stream=stream):
            for r in range(n):
                plan.execute(ins_a if r % 2 == 0 else ins_b, out, stream=stream)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(3):
        with torch.cuda.stream(stream):
            a.record(stream)
            g.replay()
            b.record(stream)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1e3 / n)
    return statistics.median(ts)


def run(args):
    import torch
    from paper_conf_micro_leebsro14_b200 import npp
    from synth import gen

    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    lim = npp.limits_query(0)
    stream = torch.cuda.Stream(device=dev)
    shapes = SHAPES if not args.shapes else [tuple(int(v) for v in s.split("x")) for s in args.shapes.split(",")]
    result = {"device": torch.cuda.get_device_name(0), "limits": lim, "rows": []}
    os.makedirs(os.path.dirname(os.path.abspath(args.out)), exist_ok=True)
    log = open(args.out + "l", "w")  # <out>l: one JSON row per measured mapping
    from oracle import sums
    for (R, C) in shapes:
        ma = gen.uniform_f32(3, (R, C), device=dev)
        mb = gen.uniform_f32(4, (R, C), device=dev)
        ma_np = ma.cpu().numpy()
        for pattern in ("SUM_ROWS", "SUM_COLS"):
            want = sums.sum_rows(ma_np) if pattern == "SUM_ROWS" else sums.sum_cols(ma_np)  # U[0,1): Σ|terms| = sum
            nbytes = R * C * 4 + (R if pattern == "SUM_ROWS" else C) * 4
            cands = npp.enumerate_mappings(pattern, (R, C), "f32", lim)
            entries = [("candidate", c) for c in cands]
            for strat in ("AUTO", "LITERAL", "TB_T", "WARP", "1D"):
                entries.append((strat, None))
            t_shape = time.perf_counter()
            for kind, rec in entries:
                if rec is None:
                    plan = npp.Plan(pattern, (R, C), "f32", kind, device=dev)
                else:
                    plan = npp.Plan(pattern, (R, C), "f32", mapping=rec, device=dev)
                out = plan.new_out()
                with torch.cuda.stream(stream):
                    plan.execute([ma], out, stream=stream)
                torch.cuda.synchronize()
                valid = bool(np.all(np.abs(out.cpu().numpy().astype(np.float64) - want) <= 1e-5 * want))
                us = time_plan(torch, plan, [ma], [mb], out, stream) if valid else float("nan")
                m = plan.mapping
                row = {
                    "pattern": pattern, "shape": [R, C], "kind": kind, "score": m["score"], "dop": m["dop"],
                    "grid": m["grid"], "block": m["block"], "mapping": brief(m), "staged": m["staged"],
                    "valid": valid, "us": round(us, 2),
                    "GB/s": round(nbytes / (us * 1e-6) / 1e9, 1) if valid else 0.0}
                result["rows"].append(row)
                log.write(json.dumps(row) + "\n")  # incremental: a cut-off run keeps what it measured
                log.flush()
                del plan, out
            print(f"{pattern} {R}x{C}: {len(entries)} mappings in {time.perf_counter() - t_shape:.1f} s",
                  flush=True)
        del ma, mb
        torch.cuda.empty_cache()
    if args.kmeans:
        sweep_kmeans(torch, npp, gen, dev, lim, stream, result, log, args)
    with open(args.out, "w") as f:
        json.dump(result, f)
    print(summarize(result))


KM_SHAPE = (1 << 16, 64, 32)  # config 4's D and K; N reduced so the slowest mappings finish in seconds


def sweep_kmeans(torch, npp, gen, dev, lim, stream, result, log, args, per_band=25):
    """The three-level nest (k-means assignment): a score-stratified sample of the Algorithm 1 candidates
    without Split (the direct executor's space), each validated against the oracle, then timed; AUTO and
    LITERAL as markers. Validation is exact equality of the assignments."""
    import random

    from oracle import kmeans as okm
    N, D, K = KM_SHAPE
    xa, c = gen.kmeans_inputs(N, D, K, device=dev)
    xb, _ = gen.kmeans_inputs(N, D, K, row_offset=N, device=dev)
    want = okm.assign(xa.cpu().numpy(), c.cpu().numpy())
    nbytes = N * D * 4 + K * D * 4 + N * 4
    cands = [r for r in npp.enumerate_mappings("KMEANS_ASSIGN", KM_SHAPE, "f32", lim)
             if not any(l["span"] == 3 for l in r["levels"])]
    rng = random.Random(17)
    bands = {}
    for r in cands:
        bands.setdefault(r["score"], []).append(r)
    sample = []
    for sc in sorted(bands):
        rng.shuffle(bands[sc])
        sample += bands[sc][:per_band]
    entries = [("candidate", r) for r in sample] + [("AUTO", None), ("LITERAL", None)]
    t0 = time.perf_counter()
    for kind, rec in entries:
        plan = (npp.Plan("KMEANS_ASSIGN", KM_SHAPE, "f32", kind, device=dev) if rec is None
                else npp.Plan("KMEANS_ASSIGN", KM_SHAPE, "f32", mapping=rec, device=dev))
        out = plan.new_out()
        with torch.cuda.stream(stream):
            plan.execute([xa, c], out, stream=stream)
        torch.cuda.synchronize()
        valid = bool(np.array_equal(out.cpu().numpy(), want))
        us = time_plan(torch, plan, [xa, c], [xb, c], out, stream) if valid else float("nan")
        m = plan.mapping
        row = {"pattern": "KMEANS_ASSIGN", "shape": list(KM_SHAPE), "kind": kind, "score": m["score"],
               "dop": m["dop"], "grid": m["grid"], "block": m["block"], "mapping": brief(m), "staged": m["staged"],
               "valid": valid, "us": round(us, 2), "GB/s": round(nbytes / (us * 1e-6) / 1e9, 1) if valid else 0.0,
               "TFLOP/s": round(2 * N * K * D / (us * 1e-6) / 1e12, 2) if valid else 0.0}
        result["rows"].append(row)
        log.write(json.dumps(row) + "\n")
        log.flush()
    print(f"KMEANS_ASSIGN {KM_SHAPE}: {len(entries)} mappings of {len(cands)} without Split "
          f"in {time.perf_counter() - t0:.1f} s", flush=True)


def _spearman(xs, ys):
    def ranks(v):
        order = sorted(range(len(v)), key=lambda i: v[i])
        r = [0.0] * len(v)
        i = 0
        while i < len(v):
            j = i
            while j + 1 < len(v) and v[order[j + 1]] == v[order[i]]:
                j += 1
            for k in range(i, j + 1):
                r[order[k]] = (i + j) / 2.0
            i = j + 1
        return r
    rx, ry = ranks(xs), ranks(ys)
    mx, my = statistics.fmean(rx), statistics.fmean(ry)
    num = sum((a - mx) * (b - my) for a, b in zip(rx, ry))
    den = (sum((a - mx) ** 2 for a in rx) * sum((b - my) ** 2 for b in ry)) ** 0.5
    return num / den if den else 0.0


def calibrate(rows):
    """Refit the intrinsic weights (G3: W_C coalescing, W_B minimum block size; P:L1402-1411 asks for
    tuning them from measurements): for each nest, recompute every timed candidate's soft-constraint
    score under a grid of (W_C, W_B) with the oracle's score terms and report the Spearman rank
    correlation of score and measured speed, and whether the top-scoring mapping would change."""
    from oracle import select as S
    lim = S.B200
    grid = [(wc, wb) for wc in (1, 2, 4, 8, 16, 32, 64) for wb in (0, 1, 2, 4, 8)]
    out = ["| nest | (W_C, W_B) | Spearman(score, speed) | time of the top-scored mapping / fastest time |",
           "|---|---|---|---|"]
    keys = []
    for r in rows:
        k = (r["pattern"], tuple(r["shape"]))
        if k not in keys:
            keys.append(k)
    for pattern, shape in keys:
        cand = [r for r in rows if (r["pattern"], tuple(r["shape"])) == (pattern, shape) and
                r["kind"] == "candidate" and r.get("valid", True) and r["us"] == r["us"]]
        if len(cand) < 3:
            continue
        nest = S.build_nest(pattern, shape)
        speed = [-r["us"] for r in cand]
        best = min(r["us"] for r in cand)
        res = []
        for wc, wb in grid:
            S.W_C, S.W_B = wc, wb
            sc = [S.score(nest, lim, _dims(r), _blocks(r)) for r in cand]
            top = max(range(len(cand)), key=lambda i: (sc[i], -cand[i]["us"]))
            res.append(((wc, wb), _spearman(sc, speed), cand[top]["us"] / best))
        S.W_C, S.W_B = 8, 1
        cur = next(x for x in res if x[0] == (8, 1))
        fit = max(res, key=lambda x: (x[1], -x[2]))
        for tag, (w, rho, ratio) in (("current", cur), ("best fit", fit)):
            out.append(f"| {pattern.lower()}{list(shape)} | {tag} {w} | {rho:.3f} | {ratio:.2f} |")
    return "\n".join(out)


def _dims(r):
    return tuple("xyz".index(tok[0]) for tok in r["mapping"].split())


def _blocks(r):
    return tuple(int(re.match(r"[xyz](\d+)", tok).group(1)) for tok in r["mapping"].split())


def summarize(result):
    rows = result["rows"]
    keys = []
    for r in rows:
        k = (r["pattern"], tuple(r["shape"]))
        if k not in keys:
            keys.append(k)
    n_bad = sum(1 for r in rows if not r.get("valid", True))
    lines = [f"validated against the oracle: {len(rows) - n_bad} of {len(rows)} mappings correct", "",
             "| nest | candidates | best candidate GB/s (score, mapping) | LITERAL GB/s (score) | LITERAL rank | "
             "AUTO GB/s | TB/T | warp | 1D | Spearman(score, GB/s) | false negatives (C) |",
             "|---|---|---|---|---|---|---|---|---|---|---|"]
    for pattern, shape in keys:
        sel = [r for r in rows if r["pattern"] == pattern and tuple(r["shape"]) == shape]
        cand = [r for r in sel if r["kind"] == "candidate" and r.get("valid", True)]
        mk = {r["kind"]: r for r in sel if r["kind"] != "candidate"}
        if not cand:
            continue
        best = max(cand, key=lambda r: r["GB/s"])
        top_score = max(r["score"] for r in cand)
        lit = mk.get("LITERAL")
        rank = f"{1 + sum(1 for r in cand if r['GB/s'] > lit['GB/s'])}/{len(cand)}" if lit else "—"
        rho = _spearman([r["score"] for r in cand], [r["GB/s"] for r in cand])
        fneg = sum(1 for r in cand if r["score"] < top_score // 2 and r["GB/s"] >= 0.9 * best["GB/s"])
        g = lambda k: mk[k]["GB/s"] if k in mk else "—"  # noqa: E731
        lines.append(
            f"| {pattern.lower()}[{shape[0]}x{shape[1]}] | {len(cand)} | {best['GB/s']} ({best['score']}, "
            f"{best['mapping']}) | {g('LITERAL')} ({lit['score'] if lit else '—'}) | {rank} | {g('AUTO')} | "
            f"{g('TB_T')} | {g('WARP')} | {g('1D')} | {rho:.2f} | {fneg} |")
    return "\n".join(lines)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/fig17.json")
    ap.add_argument("--shapes", default="")
    ap.add_argument("--summarize", default="")
    ap.add_argument("--kmeans", action="store_true", help="also sweep the k-means nest (direct executor)")
    ap.add_argument("--calibrate", default="", help="fit W_C/W_B to a sweep's jsonl (no GPU)")
    a = ap.parse_args()
    if a.calibrate:
        print(calibrate([json.loads(l) for l in open(a.calibrate) if l.strip()]))
    elif a.summarize:
        if a.summarize.endswith(".jsonl"):
            print(summarize({"rows": [json.loads(l) for l in open(a.summarize) if l.strip()]}))
        else:
            print(summarize(json.load(open(a.summarize))))
    else:
        run(a)

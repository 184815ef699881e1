"""Fig 16 of the paper on B200: the cost of the weighted sums' inner allocation (§VI-F,
P:L1289-1356; §V-A).

sumWeightedRows / sumWeightedCols (Fig 15) under the LITERAL mapping (Algorithm 1 + ControlDOP), with
the zipWith result kept in
  malloc    a device malloc per outer iteration (the code before §V-A),
  prealloc  one preallocated [outer x inner] buffer, row-major (offset m*N, stride 1) — "w/o layout opt",
  layout    the preallocated buffer laid out for the mapping (Fig 11) — the paper's fully optimised code,
and AUTO (this build: the product reduced in registers from TMA-staged tiles, no allocation at all).
Times are normalised to `layout`, as in Fig 16.

    python tools/fig16.py [--shapes 8192x8192,...] [--out gpurun_out/fig16.json]
    python tools/fig16.py --summarize gpurun_out/fig16.json
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

PAPER = {"SUM_WEIGHTED_COLS": {"malloc": 20.8, "prealloc": 5.3, "layout": 1.0},
         "SUM_WEIGHTED_ROWS": {"malloc": 16.2, "prealloc": 1.0, "layout": 1.0}}


def run(args):
    import torch
    from paper_conf_micro_leebsro14_b200 import npp
    from sweep_fig17 import brief, time_plan
    from synth import gen
    dev = torch.device("cuda:0")
    stream = torch.cuda.Stream(device=dev)
    rows_out = []
    for shp in args.shapes.split(","):
        R, C = (int(v) for v in shp.split("x"))
        ma, mb = gen.uniform_f32(3, (R, C), device=dev), gen.uniform_f32(4, (R, C), device=dev)
        for pattern in ("SUM_WEIGHTED_ROWS", "SUM_WEIGHTED_COLS"):
            rows = pattern == "SUM_WEIGHTED_ROWS"
            v = gen.uniform_f32(8, (C if rows else R,), device=dev, lo=-1.0, scale=2.0)
            M, N = (R, C) if rows else (C, R)
            lit = npp.Plan(pattern, (R, C), "f32", "LITERAL", device=dev).mapping
            variants = [("malloc", dict(lit, temp=npp.TEMP_MALLOC, temp_stride=[0, 1])),
                        ("prealloc", dict(lit, temp_stride=[N, 1])),
                        ("layout", dict(lit)), ("AUTO", None)]
            res = {}
            for name, rec in variants:
                plan = (npp.Plan(pattern, (R, C), "f32", "AUTO", device=dev) if rec is None
                        else npp.Plan(pattern, (R, C), "f32", mapping=rec, device=dev))
                out = plan.new_out()
                us = time_plan(torch, plan, [ma, v], [mb, v], out, stream, budget_ms=1500.0)
                res[name] = us
                rows_out.append({"pattern": pattern, "shape": [R, C], "variant": name, "us": round(us, 2),
                                 "mapping": brief(plan.mapping), "temp": plan.mapping["temp"],
                                 "temp_stride": plan.mapping["temp_stride"]})
                print(pattern, R, C, name, round(us, 1), "us", flush=True)
                del plan, out
            for r in rows_out:
                if r["pattern"] == pattern and r["shape"] == [R, C]:
                    r["norm"] = round(r["us"] / res["layout"], 2)
        del ma, mb
        torch.cuda.empty_cache()
    result = {"device": torch.cuda.get_device_name(0), "rows": rows_out, "paper": PAPER}
    os.makedirs(os.path.dirname(os.path.abspath(args.out)), exist_ok=True)
    json.dump(result, open(args.out, "w"), indent=1)
    print(summarize(result))


def summarize(result):
    lines = ["| nest | malloc | prealloc (row-major) | prealloc + layout (Fig 11) | AUTO (no allocation) | paper (K20c) |",
             "|---|---|---|---|---|---|"]
    keys = []
    for r in result["rows"]:
        k = (r["pattern"], tuple(r["shape"]))
        if k not in keys:
            keys.append(k)
    for pattern, shape in keys:
        sel = {r["variant"]: r for r in result["rows"] if r["pattern"] == pattern and tuple(r["shape"]) == shape}
        p = result["paper"][pattern]
        cells = [f"{sel[v]['norm']} ({sel[v]['us']:.0f} µs)" for v in ("malloc", "prealloc", "layout", "AUTO")]
        lines.append(f"| {pattern.lower()}[{shape[0]}x{shape[1]}] | " + " | ".join(cells) +
                     f" | {p['malloc']} / {p['prealloc']} / {p['layout']} |")
    return "\n".join(lines)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--shapes", default="8192x8192,65536x1024,1024x65536")
    ap.add_argument("--out", default="gpurun_out/fig16.json")
    ap.add_argument("--summarize", default="")
    a = ap.parse_args()
    if a.summarize:
        print(summarize(json.load(open(a.summarize))))
    else:
        run(a)

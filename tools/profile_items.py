"""Execute each item of a bench workload once, in order, after a warm-up — for ncu launch lists.

    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
        -k regex:npp_ --csv --log-file gpurun_out/items.csv python tools/profile_items.py paper
    python tools/profile_items.py --parse gpurun_out/items.csv paper > profiles/ncu_traffic.json
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def build(workload):
    import torch
    import bench
    from paper_conf_micro_leebsro14_b200 import npp
    from synth import gen
    dev = torch.device("cuda:0")
    items, _, _ = bench.WORKLOADS[workload](npp, gen, torch, 0, 1, "AUTO", dev)
    return torch, items


def run(workload, warm=2):
    torch, items = build(workload)
    for it in items:  # warm-up: plan setup, tensor maps, first touch
        it.run(torch.cuda.current_stream())
    torch.cuda.synchronize()
    for _ in range(warm):
        for it in items:
            it.run(torch.cuda.current_stream())
    torch.cuda.synchronize()
    print(json.dumps([it.name for it in items]))


def parse(path, workload, warm=2):
    rows = [r for r in csv.reader(l for l in open(path) if not l.startswith("=="))]
    hdr = rows[0]
    ii, mi, vi = hdr.index("ID"), hdr.index("Metric Name"), hdr.index("Metric Value")
    per = {}
    for r in rows[1:]:
        per.setdefault(int(r[ii]), {})[r[mi]] = float(r[vi].replace(",", ""))
    names = NAMES[workload]
    ids = sorted(per)
    n = len(names)
    out = {}
    last = ids[-n:]  # the final pass over the items
    for name, i in zip(names, last):
        m = per[i]
        out[name] = int(m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0))
        out[name + "/ncu_us"] = round(m.get("gpu__time_duration.sum", 0) / 1e3, 2)
    return out


NAMES = {
    "paper": ["sum_rows[64K,1K]", "sum_cols[64K,1K]", "sum_rows[8K,8K]", "sum_cols[8K,8K]", "sum_rows[1K,64K]",
              "sum_cols[1K,64K]"],
    "kmeans": ["kmeans_assign[4M,64,32]"],
    "sumcols_1m4k": ["sum_cols[1M,4K]"],
    "logreg": ["logreg_grad[16M,256]"],
    "kmeans_update": ["kmeans_update[4M,64,32]"],
    "pagerank": ["pagerank[4M,63M]"],
    "rowscols": ["sum_rows_cols[64K,1K]", "sum_rows_cols[8K,8K]", "sum_rows_cols[1K,64K]"],
}

if __name__ == "__main__":
    if sys.argv[1] == "--parse":
        print(json.dumps(parse(sys.argv[2], sys.argv[3]), indent=1))
    else:
        run(sys.argv[1])

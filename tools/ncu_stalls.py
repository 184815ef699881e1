"""Stall-reason breakdown by SASS region from an `ncu --page source --csv --print-source sass` export.
    python tools/ncu_stalls.py SRC.csv [UNITS]   (UNITS: divide executed counts, e.g. warp-tiles)
Regions are runs of consecutive instructions with the same execution count. Measurement tool only."""
import collections
import csv
import sys


def main():
    rows = list(csv.reader(open(sys.argv[1])))
    units = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
    hdr, data = rows[1], rows[2:]
    ei = hdr.index("Instructions Executed")
    reasons = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
    idx = [hdr.index(h) for h in reasons]
    tot = collections.Counter()
    regions = []
    prev, cur = None, None
    for r in data:
        e = int(r[ei] or 0)
        if e != prev:
            cur = {"exec": e, "n": 0, "st": collections.Counter()}
            regions.append(cur)
            prev = e
        cur["n"] += 1
        for h, i in zip(reasons, idx):
            v = int(r[i] or 0)
            cur["st"][h] += v
            tot[h] += v
    print("all:", ", ".join(f"{k[6:]}={v}" for k, v in tot.most_common(10)))
    for g in regions:
        s = sum(g["st"].values())
        if s < 0.02 * sum(tot.values()):
            continue
        print(f"n={g['n']:4d} exec/unit={g['exec'] / units:7.2f} samples={s:6d}: " +
              ", ".join(f"{k[6:]}={v}" for k, v in g["st"].most_common(6)))


if __name__ == "__main__":
    main()

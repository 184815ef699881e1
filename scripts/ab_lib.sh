#!/bin/bash
# A/B of two prebuilt libraries on the paper step's per-shape timings (GPU box):
#   [BENCH_ARGS="--workload rowscols"] scripts/ab_lib.sh OUTDIR LIB_B   (A = the in-tree libnpp.so; two rounds)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/$1; B=$2; mkdir -p $O
for rep in 1 2; do for name in a b; do
  if [ $name = a ]; then L=""; else L="NPP_LIB_PATH=$B"; fi
  env $L timeout 300 python bench.py --steps 20 --no-cpu --no-e2e --no-per-config --no-mappings ${BENCH_ARGS} > $O/b_$name.json 2>/dev/null
  python - $O/b_$name.json $name $rep <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read())
print("==", sys.argv[2], sys.argv[3], "step", d["value"])
for k, v in d["per_shape"].items():
    print(f"  {k:20s} {v['us']:7.2f} {v['us_pdl']:7.2f} {v['us_overlapped']:7.2f}  {v['GB/s']:8.1f}")
PY
done; done

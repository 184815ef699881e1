#!/bin/bash
# A/B of staged-sum build variants (compile-time knobs, e.g. -DNPP_TMA_STAGES=6), GPU box:
#   tools/sum_variants.sh OUTDIR "NAME:-DFLAG ..." ...   -> per-shape us (no PDL) / us_pdl / us_overlapped
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/$1; shift
mkdir -p "$O" build/variants
for spec in "base:" "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  lib=build/variants/libnpp_$name.so
  python -m paper_conf_micro_leebsro14_b200.build $flags --out=$lib > /dev/null 2>&1 || { echo "$name build failed"; continue; }
  NPP_LIB_PATH=$PWD/$lib timeout 300 python bench.py --steps 20 --no-cpu --no-e2e --no-per-config --no-mappings ${BENCH_ARGS} \
    > "$O/bench_$name.json" 2> "$O/bench_$name.err"
  python - "$O/bench_$name.json" "$name" >> "$O/sum_variants.log" <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read())
print("==", sys.argv[2], "step", d["value"])
for k, v in d["per_shape"].items():
    print(f"  {k:20s} {v['us']:7.2f} {v['us_pdl']:7.2f} {v['us_overlapped']:7.2f}  {v['GB/s']:8.1f}")
PY
done
cat "$O/sum_variants.log"

#!/bin/bash
# A/B of KMEANS_ASSIGN build variants (compile-time measurement knobs of kern_kmeans.cu), GPU box:
#   tools/km_variants.sh OUTDIR "NAME:-DFLAG ..." ...
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/$1; shift
mkdir -p "$O"
for spec in "base:" "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  lib=build/variants/libnpp_$name.so
  mkdir -p build/variants
  python -m paper_conf_micro_leebsro14_b200.build $flags --out=$lib > /dev/null 2>&1 || { echo "$name build failed"; continue; }
  echo "== $name ($flags)" >> "$O/km_variants.log"
  NPP_LIB_PATH=$PWD/$lib timeout 300 python tools/time_kmeans.py >> "$O/km_variants.log" 2>&1
done
cat "$O/km_variants.log"

#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for v in km_s2 km_s3 km_s4_r64 km_s2_d128r64; do
  if [ $v = base ]; then L=paper_conf_micro_leebsro14_b200/libnpp.so; else L=build/lib$v.so; fi
  echo "== $v"; NPP_LIB_PATH=$L timeout 300 python tools/time_kmeans.py 2>&1 | head -6
done

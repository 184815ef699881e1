#!/bin/bash
# pool divisor sweep on sum_cols[64K,1K] (Ti = 2048, unit 4), two passes
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/div64k
for pass in 1 2; do for D in 8 4 6 12 16 24 32; do
  echo "== pass=$pass div=$D $(NPP_POOL_DIV=$D timeout 120 python tools/time_plans.py --iters 40 --shapes 65536x1024 --patterns SUM_COLS 2>&1 | grep -E '^SUM_COLS ' | awk '{print $1, $2, $5, $13}')"
done; done > gpurun_out/div64k/sweep.log 2>&1
cat gpurun_out/div64k/sweep.log

#!/bin/bash
# pool divisor / unit sweep on sum_cols[8K,8K] (the dominant kernel of the paper step)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/pool8k
for D in 8 4 6 12 16 32; do for U in 1 2 4 8; do
  echo "== div=$D unit=$U"; NPP_POOL_DIV=$D NPP_POOL_UNIT=$U timeout 120 python tools/time_plans.py --iters 40 --shapes 8192x8192 --patterns SUM_COLS 2>&1 | tail -1
done; done > gpurun_out/pool8k/sweep.log 2>&1
cat gpurun_out/pool8k/sweep.log

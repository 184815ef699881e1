#!/bin/bash
# pool-unit sweep around 8 on sum_cols[8K,8K] (div 8), three passes
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/unit8k
for pass in 1 2 3; do for U in 6 8 10 12; do
  echo "== pass=$pass unit=$U $(NPP_POOL_UNIT=$U timeout 120 python tools/time_plans.py --iters 40 --shapes 8192x8192 --patterns SUM_COLS 2>&1 | grep -E '^SUM_COLS ' | awk '{print $1, $2, $5, $13}')"
done; done > gpurun_out/unit8k/sweep.log 2>&1
cat gpurun_out/unit8k/sweep.log

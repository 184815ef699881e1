#!/bin/bash
# pool-unit sweep (div 8) over the six paper shapes, two passes each
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/unit
for pass in 1 2; do for U in 4 8 16 32; do
  echo "== pass=$pass unit=$U"; NPP_POOL_UNIT=$U timeout 200 python tools/time_plans.py --iters 40 2>&1 | grep -E "^SUM_(ROWS|COLS) " | awk '{print $1, $2, $5, $13}'
done; done > gpurun_out/unit/sweep.log 2>&1
cat gpurun_out/unit/sweep.log

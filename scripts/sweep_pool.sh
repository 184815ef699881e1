#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for L in 0 1 2; do
  if [ $L = default ]; then unset NPP_DEBUG_CLAIM; else export NPP_DEBUG_CLAIM=$L; fi
  echo "== L=$L"; python tools/time_plans.py --iters 30 2>&1 | awk '{print $1, $2, $13, $15}'
done
unset NPP_DEBUG_CLAIM
NPP_DEBUG_TIMES=1 python tools/dbg_times.py 2>&1 | grep npp | awk "NR%4==0"

#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for cl in 2 4 8; do for tail in 0 150 600; do
  echo "== CL=$cl TAIL=$tail"; NPP_DEBUG_CLAIM=$cl NPP_DEBUG_TAIL=$tail python tools/time_plans.py --iters 30 2>&1 | awk '{print $1, $2, $13, $15}'
done; done

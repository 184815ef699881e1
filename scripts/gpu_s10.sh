#!/bin/bash
# weighted staged + S10 temp modes: gpu tests, Fig 16 experiment, compute-sanitizer passes
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/s10
O=gpurun_out/s10
timeout 1200 python -m pytest tests/test_gpu_sums.py -m gpu -x -q > $O/pytest_sums.log 2>&1; echo "pytest rc=$?" >> $O/pytest_sums.log
tail -3 $O/pytest_sums.log
timeout 1200 python tools/fig16.py --out $O/fig16.json > $O/fig16.log 2>&1; tail -8 $O/fig16.log
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > $O/sanitizer_$tool.log 2>&1
  echo "$tool rc=$?" >> $O/sanitizer_$tool.log; tail -4 $O/sanitizer_$tool.log
done
NPP_DEBUG_TIMES=1 timeout 300 python tools/dbg_times.py > $O/dbg_times.log 2>&1

#!/bin/bash
# re-entry check: full gpu tests, smoke, S10 / Fig 16 experiment, compute-sanitizer passes
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r01f
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -3 $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
tail -2 $O/smoke.log
timeout 1200 python tools/fig16.py --out $O/fig16.json > $O/fig16.log 2>&1; tail -12 $O/fig16.log
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > $O/sanitizer_$tool.log 2>&1
  echo "$tool rc=$?" >> $O/sanitizer_$tool.log; tail -4 $O/sanitizer_$tool.log
done

#!/bin/bash
# compute-sanitizer passes over every kernel family incl. RC, KU, PR
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/san2
mkdir -p $O
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > $O/sanitizer_$tool.log 2>&1
  echo "$tool rc=$?" >> $O/sanitizer_$tool.log; tail -3 $O/sanitizer_$tool.log
done
grep -h "Race reported\|Error" $O/sanitizer_racecheck.log | grep -o "in [a-z_]*\.cu:[0-9]*" | sort | uniq -c

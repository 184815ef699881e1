#!/bin/bash
# compute-sanitizer passes over every kernel family after the pool unit 8 rule
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/san4
mkdir -p $O
for t in memcheck racecheck synccheck; do
  timeout 420 compute-sanitizer --tool $t --error-exitcode 9 python tools/sanitize_run.py > $O/sanitizer_$t.log 2>&1
  echo "$t rc=$?" >> $O/sanitizer_$t.log; tail -2 $O/sanitizer_$t.log
done

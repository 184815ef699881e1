#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/san3
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_sums.py -m gpu -q > $O/pytest_sums.log 2>&1; echo "pytest rc=$?" >> $O/pytest_sums.log; tail -2 $O/pytest_sums.log
timeout 1200 compute-sanitizer --tool racecheck --error-exitcode 9 python tools/sanitize_run.py > $O/sanitizer_racecheck.log 2>&1
echo "racecheck rc=$?" >> $O/sanitizer_racecheck.log; tail -3 $O/sanitizer_racecheck.log
timeout 900 python bench.py --no-mappings --no-cpu --no-e2e --steps 30 > $O/bench.json 2> $O/bench.err
python -c "
import json
d=json.load(open('$O/bench.json'))
print(d['value'], ' '.join(f\"{k}:{v['GB/s']}/{v['GB/s_overlapped']}\" for k,v in d['per_shape'].items()))
"

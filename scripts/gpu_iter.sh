#!/bin/bash
# iteration pass: selected gpu tests + bench (BENCH_ARGS) + block timing stamps
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest ${TESTS:-tests/test_gpu_sums.py} -m gpu -x -q > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
timeout 600 python bench.py ${BENCH_ARGS:---no-mappings --no-cpu --no-e2e} > gpurun_out/bench_iter.json 2> gpurun_out/bench_iter.err
if [ -n "$DBG" ]; then NPP_DEBUG_TIMES=1 timeout 300 python tools/dbg_times.py > gpurun_out/dbg_times.log 2>&1; fi
tail -3 gpurun_out/pytest_iter.log
python - <<'PY'
import json
try:
    d = json.loads(open("gpurun_out/bench_iter.json").read().strip().splitlines()[-1])
    print("value", d["value"], d["unit"], "frac", d["roofline"]["frac"], d["clocks"])
    for k, v in d["per_shape"].items():
        print(" ", k, v["GB/s"], v["us"], v.get("GB/s_overlapped"), v.get("us_overlapped"))
except Exception as e:
    print("bench parse failed", e); print(open("gpurun_out/bench_iter.err").read()[-2000:])
PY

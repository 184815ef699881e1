#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sums.py -m gpu -x -q > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
tail -2 gpurun_out/pytest_iter.log
NPP_DEBUG_TIMES=1 timeout 300 python tools/dbg_times.py > gpurun_out/dbg_times.log 2>&1
show() {
  python - "$1" <<'PY'
import json, sys
d = json.loads(open(f"gpurun_out/sweep_{sys.argv[1]}.json").read().strip().splitlines()[-1])
print(sys.argv[1], "value", d["value"], " ".join(f"{v['us']}/{v.get('us_overlapped')}" for v in d["per_shape"].values()))
PY
}
for i in 1 2; do
timeout 300 python bench.py --no-mappings --no-cpu --no-e2e --steps 30 > gpurun_out/sweep_new.json 2>/dev/null; show new
NPP_LIB_PATH=build/libnpp_prev.so timeout 300 python bench.py --no-mappings --no-cpu --no-e2e --steps 30 > gpurun_out/sweep_prev.json 2>/dev/null; show prev
done

#!/bin/bash
# A/B: HEAD static kernel vs pool/PDL variants, bench per-shape times (serialised/overlapped)
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
run() {  # tag lib div unit
  NPP_LIB_PATH=$2 NPP_POOL_DIV=$3 NPP_POOL_UNIT=$4 timeout 300 python bench.py --no-mappings --no-cpu --no-e2e --steps 30 > gpurun_out/sweep_$1.json 2>/dev/null
  show $1
}
(cd build/head && timeout 300 python bench.py --no-mappings --no-cpu --no-e2e --steps 30 > ../../gpurun_out/sweep_head.json 2>/dev/null); show head
L=paper_conf_micro_leebsro14_b200/libnpp.so
S3=build/libnpp_s3.so
run s4_d8_u4 $L 8 4
run s4_d8_u2 $L 8 2
run s4_d1e6 $L 1000000 4
run s3_d8_u4 $S3 8 4
run s3_d1e6 $S3 1000000 4
(cd build/head && timeout 300 python bench.py --no-mappings --no-cpu --no-e2e --steps 30 > ../../gpurun_out/sweep_head.json 2>/dev/null); show head
run s4_d8_u4 $L 8 4

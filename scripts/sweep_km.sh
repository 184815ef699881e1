#!/bin/bash
# k-means variant sweep: R rounds over the libraries (interleaved, so drift hits all alike), then
# the kmeans parity tests on the default library
cd "${GRAFT_REPO_ROOT:-/root/repo}"
R=${R:-3}
for r in $(seq $R); do
  for L in paper_conf_micro_leebsro14_b200/libnpp.so "$@"; do
    echo -n "$r $L "; NPP_LIB_PATH=$PWD/$L python bench.py --workload kmeans --steps 10 --warmup 3 --no-cpu --no-e2e 2>&1 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().split(chr(10))[-1]); r=d['roofline']; print(r['duration_us'], r['achieved'], r['frac'])"
  done
done
timeout 600 python -m pytest tests/test_gpu_nests.py -x -q -k kmeans 2>&1 | tail -1

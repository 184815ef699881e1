#!/bin/bash
# re-entry check: gpu tests, smoke, bench (paper + kmeans) on the current tree
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --workload kmeans --steps 10 --warmup 3 --no-mappings > gpurun_out/bench_kmeans.json 2> gpurun_out/bench_kmeans.err
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log

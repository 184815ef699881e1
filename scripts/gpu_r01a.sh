#!/bin/bash
# round-1 first GPU pass: smoke, gpu tests, bench, ncu launch list + full capture of the sum kernels
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
nproc > gpurun_out/nproc.txt; lscpu | grep "Model name" >> gpurun_out/nproc.txt
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:npp_ --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-mappings --no-cpu --no-e2e > gpurun_out/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_sum -s 18 -c 6 -o gpurun_out/prof_sum python bench.py --steps 1 --warmup 3 --no-mappings --no-cpu --no-e2e > gpurun_out/b_ncu_full.log 2>&1
echo done

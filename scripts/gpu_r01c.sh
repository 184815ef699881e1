#!/bin/bash
# round-1 profiling pass: gpu tests, bench (all workloads), ncu launch lists + full captures
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
for w in kmeans logreg sumcols_1m4k; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for w in paper kmeans logreg; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:npp_ --csv --log-file gpurun_out/items_$w.csv python tools/profile_items.py $w > gpurun_out/items_$w.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:npp_ --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-mappings --no-cpu --no-e2e > gpurun_out/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_sum_tma -s 6 -c 6 -o gpurun_out/prof_r01_sum python tools/profile_items.py paper > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_logreg -s 1 -c 1 -o gpurun_out/prof_r01_logreg python tools/run_one.py logreg 512 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_kmeans -s 1 -c 1 -o gpurun_out/prof_r01_kmeans python tools/run_one.py kmeans > /dev/null 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log

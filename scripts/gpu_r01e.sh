#!/bin/bash
# round-1 refresh: full gpu tests, smoke, bench (all workloads + reference arm), ncu launch lists,
# per-item DRAM traffic, --set full captures of the top kernels
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/r01e
O=gpurun_out/r01e
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
for w in kmeans logreg sumcols_1m4k; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > $O/bench_$w.json 2> $O/bench_$w.err; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref.json 2> $O/bench_ref.err
for w in paper kmeans logreg; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:npp_ --csv --log-file $O/items_$w.csv python tools/profile_items.py $w > $O/items_$w.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:npp_ --csv --log-file $O/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-mappings --no-cpu --no-e2e > $O/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_sum_tma -s 6 -c 6 -o $O/prof_sum python tools/profile_items.py paper > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_logreg -s 1 -c 1 -o $O/prof_logreg python tools/run_one.py logreg 512 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_kmeans_tma -s 1 -c 1 -o $O/prof_kmeans python tools/run_one.py kmeans > /dev/null 2>&1
tail -3 $O/pytest_gpu.log; tail -2 $O/smoke.log

#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
./build/tools/micro_tiles 2>&1 | head -3 > gpurun_out/ab.txt
python tools/time_plans.py >> gpurun_out/ab.txt 2>&1
python tools/time_plans.py --dtype i32 >> gpurun_out/ab.txt 2>&1
timeout 600 ncu --set full --clock-control none -k regex:npp_sum_tma -s 3 -c 1 -o gpurun_out/prof_tma_rows python tools/time_plans.py --shapes 65536x1024 --patterns SUM_ROWS --iters 2 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:npp_sum_tma -s 3 -c 1 -o gpurun_out/prof_tma_cols python tools/time_plans.py --shapes 8192x8192 --patterns SUM_COLS --iters 2 > /dev/null 2>&1
cat gpurun_out/ab.txt

#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
./build/tools/micro_order > gpurun_out/ab2.txt 2>&1
python tools/time_plans.py >> gpurun_out/ab2.txt 2>&1
cat gpurun_out/ab2.txt

#!/bin/bash
# micro-measurements: launch gap / ramp / tail of 256 MiB streaming passes
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/micro_tail tools/micro_tail.cu > /dev/null 2>&1
timeout 300 /tmp/micro_tail > gpurun_out/micro_tail.log 2>&1
NPP_DEBUG_TIMES=1 timeout 300 python tools/dbg_times.py > gpurun_out/dbg_times.log 2>&1
cat gpurun_out/micro_tail.log

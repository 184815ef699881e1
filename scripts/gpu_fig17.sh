#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 2400 python tools/sweep_fig17.py --out gpurun_out/fig17.json > gpurun_out/fig17.log 2>&1
tail -12 gpurun_out/fig17.log

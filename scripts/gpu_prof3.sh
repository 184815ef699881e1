#!/bin/bash
# --set full captures of the current RC, KU and PR kernels
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/prof3
mkdir -p $O
timeout 600 ncu --set full --clock-control none --import-source on -k regex:npp_rowscols -s 2 -c 1 -o $O/prof_rc_8k python tools/run_one.py rowscols 8192x8192 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:npp_kmupdate -s 1 -c 1 -o $O/prof_ku python tools/profile_items.py kmeans_update > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:npp_pagerank_kernel -s 1 -c 1 -o $O/prof_pr python tools/profile_items.py pagerank > /dev/null 2>&1
ls -la $O

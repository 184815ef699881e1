O=gpurun_out/r02ag; mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -o /tmp/micro_gap tools/micro_gap.cu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k gap_kernel -s 40 -c 1 -o $O/micro_s4 /tmp/micro_gap 5 > $O/micro_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:npp_sum_tma -s 3 -c 1 -o $O/rx_wide python tools/run_one.py sumrows 65536x1024 > $O/rx_ncu.log 2>&1
for f in micro_s4 rx_wide; do ncu -i $O/$f.ncu-rep --page raw --csv > $O/${f}_raw.csv 2>/dev/null; ncu -i $O/$f.ncu-rep --page details --csv > $O/${f}_details.csv 2>/dev/null; done
ls -la $O

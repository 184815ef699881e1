# Per-launch overhead study of the staged sums (tools/micro_gap.cu, tools/sum_stamps.py), GPU box.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/${1:-gap}; mkdir -p $O build/variants
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/micro_gap tools/micro_gap.cu > /dev/null 2>&1 && timeout 300 /tmp/micro_gap > $O/micro_gap.log 2>&1
python -m paper_conf_micro_leebsro14_b200.build -DNPP_SUM_STAMPS --out=build/variants/libnpp_stamps.so > /dev/null 2>&1
NPP_LIB_PATH=$PWD/build/variants/libnpp_stamps.so timeout 300 python tools/sum_stamps.py > $O/sum_stamps.log 2>&1
python -m paper_conf_micro_leebsro14_b200.build -DNPP_SUM_NO_COMBINE --out=build/variants/libnpp_nocomb.so > /dev/null 2>&1
NPP_LIB_PATH=$PWD/build/variants/libnpp_nocomb.so timeout 300 python tools/time_plans.py --no-pdl --nbuf 8 --iters 20 > $O/plans_nopdl_nocomb.log 2>&1
cat $O/micro_gap.log $O/sum_stamps.log $O/plans_nopdl_nocomb.log

#!/bin/bash
# verify the RX one-row SUM_ROWS tiles (fd755de) and refresh the paper-step bench line + ncu evidence
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=${OUT:-gpurun_out/r01i}
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/nvsmi.txt 2>&1
timeout 300 python tools/check_r1_rows.py > $O/check_r1_rows.log 2>&1; echo "check rc=$?" >> $O/check_r1_rows.log
tail -3 $O/check_r1_rows.log
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -2 $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
tail -2 $O/smoke.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --workload rowscols --steps 10 --warmup 3 > $O/bench_rowscols.json 2> $O/bench_rowscols.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:npp_ --csv --log-file $O/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-mappings --no-cpu --no-e2e > $O/b_ncu.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:npp_ --csv --log-file $O/items_paper.csv python tools/profile_items.py paper > $O/items_paper.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_sum_tma -s 6 -c 6 -o $O/prof_sum python tools/profile_items.py paper > /dev/null 2>&1
python - <<'PY'
import json
for w in ["bench","bench_rowscols","bench_ref"]:
    try:
        d=json.load(open(''+__import__("os").environ.get("OUT","gpurun_out/r01i")+'/'+w+'.json'))
        r=d.get('roofline',{})
        print(w, d['value'], d['unit'], 'frac', r.get('frac'), 'clk', d.get('clocks',{}).get('sm_mhz'), d.get('clocks',{}).get('reasons'))
    except Exception as e:
        print(w, 'ERR', e)
PY
ls $O

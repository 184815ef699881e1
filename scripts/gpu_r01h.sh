#!/bin/bash
# final round-1 refresh: gpu tests, smoke, all bench lines, ncu launch list of the step, per-item DRAM
# traffic of every workload, --set full captures of the dominant sum kernel and the new families
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r01h
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -2 $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
tail -2 $O/smoke.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
for w in kmeans logreg sumcols_1m4k rowscols kmeans_update pagerank; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > $O/bench_$w.json 2> $O/bench_$w.err; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:npp_ --csv --log-file $O/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-mappings --no-cpu --no-e2e > $O/b_ncu.log 2>&1
for w in paper kmeans logreg rowscols kmeans_update pagerank; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:npp_ --csv --log-file $O/items_$w.csv python tools/profile_items.py $w > $O/items_$w.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:npp_sum_tma -s 6 -c 6 -o $O/prof_sum python tools/profile_items.py paper > /dev/null 2>&1
python - <<'PY'
import json
for w in ["bench","bench_kmeans","bench_logreg","bench_sumcols_1m4k","bench_rowscols","bench_kmeans_update","bench_pagerank","bench_ref"]:
    try:
        d=json.load(open('gpurun_out/r01h/'+w+'.json'))
        r=d.get('roofline',{})
        print(w, d['value'], d['unit'], 'frac', r.get('frac'), 'clk', d.get('clocks',{}).get('sm_mhz'), d.get('clocks',{}).get('reasons'))
    except Exception as e:
        print(w, 'ERR', e)
PY
ls $O

#!/bin/bash
# fused sumRows+sumCols (class RC): gpu tests, bench (rowscols workload + paper step with fused table),
# ncu items + a --set full capture of the [8K,8K] fused launch
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/rc1
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_sums.py -m gpu -q -k "rows_cols or weighted" > $O/pytest_rc.log 2>&1; echo "pytest rc=$?" >> $O/pytest_rc.log
tail -15 $O/pytest_rc.log
timeout 600 python bench.py --workload rowscols --steps 20 --warmup 3 --no-cpu > $O/bench_rowscols.json 2> $O/bench_rowscols.err; tail -3 $O/bench_rowscols.err
timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu --no-e2e > $O/bench_paper.json 2> $O/bench_paper.err; tail -3 $O/bench_paper.err
python -c "
import json
for f in ['bench_rowscols','bench_paper']:
    d=json.load(open('$O/'+f+'.json'))
    print(f, d['value'], json.dumps(d.get('per_shape'),indent=0)[:1500])
    print(json.dumps(d.get('fused_rows_cols'),indent=0))
"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:npp_ --csv --log-file $O/items_rowscols.csv python tools/profile_items.py rowscols > $O/items.log 2>&1
python tools/profile_items.py --parse $O/items_rowscols.csv rowscols
timeout 600 ncu --set full --clock-control none --import-source on -k regex:npp_rowscols -s 2 -c 1 -o $O/prof_rc_8k python tools/run_one.py rowscols 8192x8192 > /dev/null 2>&1
ls $O

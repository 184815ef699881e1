#!/bin/bash
# PageRank step (class PR): gpu tests, bench, ncu items + full capture
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/pr1
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_nests.py -m gpu -q -k "pagerank" > $O/pytest_pr.log 2>&1; echo "pytest rc=$?" >> $O/pytest_pr.log
tail -15 $O/pytest_pr.log
timeout 600 python bench.py --workload pagerank --steps 20 --warmup 3 > $O/bench_pagerank.json 2> $O/bench_pr.err; tail -3 $O/bench_pr.err
python -c "
import json
d=json.load(open('$O/bench_pagerank.json'))
print(d['value'], d['ms_per_step'], d['roofline'], d.get('cpu_baseline'), d.get('e2e'))
"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors.sum --clock-control none -k regex:npp_pagerank --csv --log-file $O/items_pr.csv python tools/profile_items.py pagerank > $O/items.log 2>&1
python tools/profile_items.py --parse $O/items_pr.csv pagerank
grep -i "lts__t_sectors" $O/items_pr.csv | tail -1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:npp_pagerank -s 1 -c 1 -o $O/prof_pr python tools/profile_items.py pagerank > /dev/null 2>&1
ls $O

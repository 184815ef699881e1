#!/bin/bash
# k-means update (class KU): gpu tests, bench, ncu items + full capture
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/ku1
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_nests.py -m gpu -q -k "update or lloyd" > $O/pytest_ku.log 2>&1; echo "pytest rc=$?" >> $O/pytest_ku.log
tail -15 $O/pytest_ku.log
timeout 600 python bench.py --workload kmeans_update --steps 20 --warmup 3 > $O/bench_kmeans_update.json 2> $O/bench_ku.err; tail -3 $O/bench_ku.err
python -c "
import json
d=json.load(open('$O/bench_kmeans_update.json'))
print(d['value'], d['ms_per_step'], d['roofline'], d.get('cpu_baseline'), d.get('e2e'))
"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:npp_kmupdate --csv --log-file $O/items_ku.csv python tools/profile_items.py kmeans_update > $O/items.log 2>&1
python tools/profile_items.py --parse $O/items_ku.csv kmeans_update
timeout 600 ncu --set full --clock-control none --import-source on -k regex:npp_kmupdate -s 1 -c 1 -o $O/prof_ku python tools/profile_items.py kmeans_update > /dev/null 2>&1
ls $O

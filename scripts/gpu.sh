#!/bin/bash
# One entry point for the GPU-box passes (run under gpurun from the repo root):
#   scripts/gpu.sh OUTDIR STEP [STEP ...]
# steps: tests  smoke  bench  bench_all  ref  launches  items  full:<kernel-regex>:<workload>  san
# Everything lands in gpurun_out/OUTDIR (merged back by gpurun; copy what is judged into profiles/).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/$1; shift
mkdir -p "$O"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > "$O/nvsmi.txt" 2>&1
for step in "$@"; do
  case "$step" in
    tests)
      eval "timeout 2400 python -m pytest ${PYTEST_PATHS:-tests} -m gpu -q ${PYTEST_ARGS}" > "$O/pytest_gpu.log" 2>&1
      echo "pytest rc=$?" >> "$O/pytest_gpu.log"; tail -3 "$O/pytest_gpu.log" ;;
    smoke)
      timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > "$O/smoke.log" 2>&1
      echo "smoke rc=$?" >> "$O/smoke.log"; tail -2 "$O/smoke.log" ;;
    bench)
      timeout 900 python bench.py ${BENCH_ARGS} > "$O/bench.json" 2> "$O/bench.err"; echo "bench rc=$?" ;;
    bench_all)
      for w in sumcols_1m4k kmeans logreg rowscols kmeans_update pagerank; do
        timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > "$O/bench_$w.json" 2> "$O/bench_$w.err"
      done ;;
    ref)
      timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > "$O/bench_ref.json" 2> "$O/bench_ref.err" ;;
    launches)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:npp_ --csv \
        --log-file "$O/launches_bench.csv" python bench.py --steps 2 --warmup 3 --no-mappings --no-cpu --no-e2e \
        --no-per-config > "$O/launches.log" 2>&1 ;;
    items)
      for w in paper sumcols_1m4k kmeans logreg rowscols kmeans_update pagerank; do
        timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
          --clock-control none -k regex:npp_ --csv --log-file "$O/items_$w.csv" \
          python tools/profile_items.py $w > "$O/items_$w.log" 2>&1
      done ;;
    full:*)  # full:<kernel-regex>:<workload>[:<skip>[:<count>]] (skip/count of the matching launches)
      IFS=: read -r _ rx wl sk ct <<< "$step"
      timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:$rx" -s "${sk:-4}" -c "${ct:-3}" \
        -o "$O/full_${wl}" python tools/profile_items.py "$wl" > "$O/full_${wl}.log" 2>&1
      ncu -i "$O/full_${wl}.ncu-rep" --page details --csv > "$O/full_${wl}_details.csv" 2>/dev/null
      ncu -i "$O/full_${wl}.ncu-rep" --page raw --csv > "$O/full_${wl}_raw.csv" 2>/dev/null ;;
    san)
      for tool in memcheck racecheck synccheck initcheck; do
        timeout 1500 compute-sanitizer --tool $tool --error-exitcode 1 python tools/sanitize_run.py \
          > "$O/san_$tool.log" 2>&1; echo "$tool rc=$?" >> "$O/san_$tool.log"; tail -1 "$O/san_$tool.log"
      done ;;
    *) echo "unknown step $step" ;;
  esac
done
ls "$O"

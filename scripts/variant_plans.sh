# A/B of staged-sum build variants on isolated (no-PDL) graph-replayed launches, GPU box:
#   scripts/variant_plans.sh OUTDIR "NAME:-DFLAG ..." ...   (the first run is the default build)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/$1; shift
mkdir -p "$O" build/variants
for rep in 1 2; do
for spec in "base:" "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  lib=build/variants/libnpp_$name.so
  [ -f $lib ] || python -m paper_conf_micro_leebsro14_b200.build $flags --out=$lib > /dev/null 2>&1 || { echo "$name build failed"; continue; }
  echo "== $name ($flags) rep $rep" >> "$O/variants.log"
  NPP_LIB_PATH=$PWD/$lib timeout 300 python tools/time_plans.py --no-pdl --nbuf 8 --iters 20 >> "$O/variants.log" 2>&1
done
done
cat "$O/variants.log"

# A/B of build variants with any timing tool, GPU box:
#   scripts/variants.sh OUTDIR TOOL "NAME:-DFLAG ..." ...   (base = the default build; two rounds)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/$1; TOOL=$2; shift 2
mkdir -p "$O" build/variants
for rep in 1 2; do
for spec in "base:" "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  lib=build/variants/libnpp_$name.so
  [ -f $lib ] || python -m paper_conf_micro_leebsro14_b200.build $flags --out=$lib > /dev/null 2>&1 || { echo "$name build failed"; continue; }
  echo "== $name ($flags) rep $rep" >> "$O/variants.log"
  NPP_LIB_PATH=$PWD/$lib timeout 300 python $TOOL >> "$O/variants.log" 2>&1
done
done
grep -v "^$" "$O/variants.log"

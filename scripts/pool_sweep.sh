cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02ab; mkdir -p $O
for cfg in "8 0" "8 4" "8 16" "16 0" "16 4" "4 0"; do
  set -- $cfg
  if [ "$2" = "0" ]; then unset NPP_POOL_UNIT; else export NPP_POOL_UNIT=$2; fi
  export NPP_POOL_DIV=$1
  timeout 300 python bench.py --steps 20 --no-cpu --no-e2e --no-per-config --no-mappings > $O/b_$1_$2.json 2>/dev/null
  python - $O/b_$1_$2.json "div=$1 unit=$2" >> $O/pool.log <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read())
print("==", sys.argv[2], "step", d["value"], " ".join(f"{k}:{v['us']}" for k, v in d["per_shape"].items() if "cols" in k))
PY
done
cat $O/pool.log

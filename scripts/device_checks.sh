#!/bin/bash
# The GPU parity suite against a -DNPP_DEVICE_CHECKS build (device-side bounds checks that trap on a
# violation): the stand-in for compute-sanitizer where the pool has it closed. GPU box:
#   scripts/device_checks.sh OUTDIR
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/$1; mkdir -p "$O" build/checks
L=build/checks/libnpp_checks.so
[ -f $L ] || python -m paper_conf_micro_leebsro14_b200.build -DNPP_DEVICE_CHECKS --out=$PWD/$L > /dev/null
NPP_LIB_PATH=$PWD/$L timeout 2400 python -m pytest tests -m gpu -q -p no:randomly > "$O/pytest_device_checks.log" 2>&1
echo "pytest rc=$?" >> "$O/pytest_device_checks.log"
NPP_LIB_PATH=$PWD/$L timeout 600 python tools/sanitize_run.py > "$O/sanitize_run_device_checks.log" 2>&1
echo "sanitize_run rc=$?" >> "$O/sanitize_run_device_checks.log"
tail -3 "$O/pytest_device_checks.log"; tail -2 "$O/sanitize_run_device_checks.log"

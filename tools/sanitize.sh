#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over smoke() (sort in
# every order, load_interpolator, advance_p TMA kernel, unload, rho) and one
# loopback single-round device-initiated exchange step (advance_p inbox
# stores, LSA barrier, migration kernels).  Logs: gpurun_out/san_*.txt
#   gpurun -- tools/sanitize.sh
cd "$(dirname "$0")/.."
CS=/usr/local/cuda/bin/compute-sanitizer
SMOKE='import __graft_entry__ as g; g.smoke()'
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 $CS --tool $tool --print-limit 50 --error-exitcode 9 python -c "$SMOKE" \
    > gpurun_out/san_smoke_$tool.txt 2>&1
  echo "smoke $tool rc=$?" | tee -a gpurun_out/san_summary.txt
done
for tool in memcheck racecheck synccheck; do
  timeout 900 $CS --tool $tool --print-limit 50 --error-exitcode 9 python tools/sanitize_loopback.py \
    > gpurun_out/san_loop_$tool.txt 2>&1
  echo "loopback $tool rc=$?" | tee -a gpurun_out/san_summary.txt
done

#!/bin/bash
# Round-2 profiles: the launch list of one bench period (ncu, serialised,
# cold-cache: SHARES, not absolute times) and ncu --set full of k_advance_tma
# for ions right after the sort (issue-bound) and electrons 19 steps later
# (L1/L2-reduction-bound), plus the sort kernels of one late sort.
cd "$(dirname "$0")/.."
set -x
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches.csv \
  python bench.py --steps 2 --warmup 1 --profile > gpurun_out/r02_prof_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_advance_tma --launch-skip 41 -c 1 \
  -o gpurun_out/r02_adv_ion_step0 python bench.py --steps 1 --warmup 1 --profile > gpurun_out/r02_prof1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_advance_tma --launch-skip 78 -c 1 \
  -o gpurun_out/r02_adv_el_step19 python bench.py --steps 1 --warmup 1 --profile > gpurun_out/r02_prof2.log 2>&1
ls -la gpurun_out

#!/bin/bash
# Dev A/B over libvpic_<name>.so builds: avg advance ms by step since sort
for n in "$@"; do
  if [ "$n" = base ]; then L=""; else L=$PWD/paper_conf_sc_tanlta25_b200/libvpic_$n.so; fi
  VPIC_LIB=$L timeout 300 python bench.py --steps ${STEPS:-2} --warmup 1 --no-cpu-baseline --no-e2e $EXTRA > gpurun_out/exp_$n.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/exp_$n.log').read().splitlines()[-1]);r=d['roofline'];s=r['avg_launch_ms_by_step_since_sort'];print('$n', round(d['value']/1e9,2), 'Gp/s adv_ms', round(r['avg_launch_ms'],3), 'step0', s[0], 'step19', s[-1], 'sort', d.get('sort_ms_by_species'))" || tail -5 gpurun_out/exp_$n.log
done

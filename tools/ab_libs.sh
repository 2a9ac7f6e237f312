#!/bin/bash
# A/B of whole libvpic builds on the default bench: alternate the libraries
# REPS times (same box), print G pushes/s, mean advance launch, sort ms, clock.
#   tools/ab_libs.sh base:paper_conf_sc_tanlta25_b200/libvpic.so exp:paper_conf_sc_tanlta25_b200/libvpic_exp.so
REPS=${REPS:-3}
for r in $(seq $REPS); do
  for nl in "$@"; do
    n=${nl%%:*}; l=${nl#*:}
    VPIC_LIB=$PWD/$l timeout 600 python bench.py --steps ${STEPS:-2} --warmup 1 --no-cpu-baseline --no-e2e $EXTRA \
      > gpurun_out/ab_$n.json 2> gpurun_out/ab_$n.err
    python -c "import json;d=json.loads(open('gpurun_out/ab_$n.json').read().splitlines()[-1]);r=d['roofline'];print('$n', round(d['value']/1e9,3), 'adv_ms', round(r['avg_launch_ms'],3), 'frac', round(r['frac'],3), 'sort', d.get('sort_ms_by_species'), 'mhz', d['clocks']['sm_mhz'])" || tail -3 gpurun_out/ab_$n.err
  done
done

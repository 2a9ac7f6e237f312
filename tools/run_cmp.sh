#!/bin/bash
# Dev: repeated bench lines into gpurun_out/res.txt.  Usage: run_cmp.sh "<label>|<VPIC_LIB or ->|<bench args>" ...
rm -f gpurun_out/res.txt
for spec in "$@"; do
  IFS='|' read -r label lib bargs <<< "$spec"
  [ "$lib" = "-" ] && lib=""
  VPIC_LIB=$lib timeout 600 python bench.py --no-cpu-baseline --no-e2e $bargs > gpurun_out/b_x.log 2>&1
  tail -1 gpurun_out/b_x.log | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$label', round(d['value']/1e9,2), 'Gp/s', round(d['ms_per_step'],1), 'ms/step adv', round(r['avg_launch_ms'],3), 'sort', d.get('sort_ms_by_species'), d['config'].get('exchange'))" >> gpurun_out/res.txt 2>&1 || tail -3 gpurun_out/b_x.log >> gpurun_out/res.txt
done
cat gpurun_out/res.txt

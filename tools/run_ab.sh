#!/bin/bash
# A/B of advance_p variants: prints Gpushes/s, avg advance launch ms, roofline frac
for k in ${KERNELS:-direct tma}; do for d in ${DEPOSITS:-warp}; do
  timeout 300 python bench.py --steps ${STEPS:-2} --warmup 1 --no-cpu-baseline --no-e2e --kernel $k --deposit $d $EXTRA > gpurun_out/bench_${k}_${d}.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/bench_${k}_${d}.log').read().splitlines()[-1]);print('$k $d', round(d['value']/1e9,2), 'Gp/s adv_ms', round(d['roofline']['avg_launch_ms'],3), 'frac', round(d['roofline']['frac'],3), 'step_ms', round(d['ms_per_step'],1))" || tail -5 gpurun_out/bench_${k}_${d}.log
done; done

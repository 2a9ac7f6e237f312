#!/bin/bash
# Fig. 7 analogue on B200: push+sort rate for each sort order (and the random order)
for o in standard strided tiled_strided; do
  timeout 300 python bench.py --steps ${STEPS:-2} --warmup 1 --no-cpu-baseline --no-e2e --order $o $EXTRA > gpurun_out/bench_order_$o.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/bench_order_$o.log').read().splitlines()[-1]);r=d['roofline'];print('$o', round(d['value']/1e9,2), 'Gp/s adv_ms', round(r['avg_launch_ms'],3), 'step_ms', round(d['ms_per_step'],1), 'by_step', r['avg_launch_ms_by_step_since_sort'][0], r['avg_launch_ms_by_step_since_sort'][-1])" || tail -3 gpurun_out/bench_order_$o.log
done
timeout 300 python bench.py --steps ${STEPS:-2} --warmup 1 --no-cpu-baseline --no-e2e --order none --shuffle $EXTRA > gpurun_out/bench_order_random.log 2>&1
python -c "import json;d=json.loads(open('gpurun_out/bench_order_random.log').read().splitlines()[-1]);r=d['roofline'];print('random', round(d['value']/1e9,2), 'Gp/s adv_ms', round(r['avg_launch_ms'],3), 'step_ms', round(d['ms_per_step'],1))" || tail -3 gpurun_out/bench_order_random.log

# AUTO deposit policy thresholds (SMEM between LO and HI cells of thermal spread)
for r in 1 2; do
for pol in "0.4 1.3" "0.3 1.3" "0.6 1.3" "0.4 1.0" "0.4 2.0" "9 9"; do
  set -- $pol
  timeout 400 python tools/gpu/bench_policy.py $1 $2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/pol.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/pol.log').read().splitlines()[-1]);r=d['roofline'];f=lambda v:[round(x,2) for x in v];print('$1-$2', round(d['value']/1e9,3), 'adv', round(r['avg_launch_ms'],3), 'e', f(r['launch_ms_by_species_step']['electron'][::2]), d['clocks']['sm_mhz'])" || tail -3 gpurun_out/pol.log
done; done

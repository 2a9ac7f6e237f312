for r in 1 2; do
for pol in "0.4 1.3" "0.1 1.3" "0.2 1.3"; do
  set -- $pol
  timeout 400 python tools/gpu/bench_policy.py $1 $2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/pol.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/pol.log').read().splitlines()[-1]);r=d['roofline'];f=lambda v:[round(x,2) for x in v];print('$1-$2', round(d['value']/1e9,3), 'adv', round(r['avg_launch_ms'],3), 'i', f(r['launch_ms_by_species_step']['ion'][::2]), d['clocks']['sm_mhz'])" || tail -3 gpurun_out/pol.log
done; done

for r in 1 2; do
for m in "" "--concurrent-species"; do
  timeout 400 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e $m > gpurun_out/conc.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/conc.log').read().splitlines()[-1]);r=d['roofline'];print('[$m]', round(d['value']/1e9,3), 'ms/period', round(d['ms_per_step'],1), 'sort', d['sort_ms_by_species'], d['clocks']['sm_mhz'])" || tail -3 gpurun_out/conc.log
done; done

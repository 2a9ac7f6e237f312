set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -3
for r in 1 2; do
for L in base new; do
  if [ $L = base ]; then export VPIC_LIB=$PWD/paper_conf_sc_tanlta25_b200/libvpic_base.so; else unset VPIC_LIB; fi
  timeout 400 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab_${L}_$r.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/ab_${L}_$r.log').read().splitlines()[-1]);r=d['roofline'];print('$L', round(d['value']/1e9,3), 'adv', round(r['avg_launch_ms'],3), 'frac', round(r['frac'],3), 'sort', d['sort_ms_by_species'], 'e', r['launch_ms_by_species_step']['electron'][:3], r['launch_ms_by_species_step']['electron'][-2:], 'i', r['launch_ms_by_species_step']['ion'][:3], r['launch_ms_by_species_step']['ion'][-2:], d['clocks']['sm_mhz'])" || tail -5 gpurun_out/ab_${L}_$r.log
done; done

# Dev A/B on one GPU: bash tools/gpu/ab.sh "<lib names: 'new' = libvpic.so, X = libvpic_X.so>" [reps] [extra bench args]
LIBS=$1; REPS=${2:-2}; EXTRA=$3
mkdir -p gpurun_out
B=$PWD/paper_conf_sc_tanlta25_b200
for r in $(seq $REPS); do
for L in $LIBS; do
  if [ $L = new ]; then unset VPIC_LIB; else export VPIC_LIB=$B/libvpic_$L.so; fi
  timeout 400 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e $EXTRA > gpurun_out/ab_${L}_$r.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/ab_${L}_$r.log').read().splitlines()[-1]);r=d['roofline'];f=lambda v:[round(x,2) for x in v];print('$L', round(d['value']/1e9,3), 'adv', round(r['avg_launch_ms'],3), 'frac', round(r['frac'],3), 'sort', d['sort_ms_by_species'], 'e', f(r['launch_ms_by_species_step']['electron'][::3]), 'i', f(r['launch_ms_by_species_step']['ion'][::3]), d['clocks']['sm_mhz'])" || tail -5 gpurun_out/ab_${L}_$r.log
done; done

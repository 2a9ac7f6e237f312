# C3 (Harris sheet) and C5 (LPI slab, 2^31 particles) bench lines with the current build
mkdir -p gpurun_out/cfg
timeout 900 python bench.py --config 2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cfg/bench_c3.json 2> gpurun_out/cfg/c3.err
timeout 1200 python bench.py --config 4 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cfg/bench_c5.json 2> gpurun_out/cfg/c5.err
for f in c3 c5; do python -c "import json;d=json.loads(open('gpurun_out/cfg/bench_$f.json').read().splitlines()[-1]);print('$f', round(d['value']/1e9,2), d['roofline']['frac'], d.get('sort_ms_by_species'), d['clocks']['sm_mhz'])" || tail -3 gpurun_out/cfg/$f.err; done

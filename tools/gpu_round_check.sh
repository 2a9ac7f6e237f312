# Round re-check on one B200: GPU tests, smoke, two default bench lines, the
# reference arm, and the ncu launch list of the bench command.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/bench1.json 2> gpurun_out/bench1.err
timeout 600 python bench.py > gpurun_out/bench2.json 2> gpurun_out/bench2.err
[ -n "$SKIP_REF" ] || timeout 600 python bench.py --impl reference --steps 1 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01_launches.csv python bench.py --steps 2 --warmup 1 --profile > gpurun_out/prof_bench.log 2>&1
tail -3 gpurun_out/gpu_tests.log; cat gpurun_out/bench1.json gpurun_out/bench2.json

# Full GPU test suite + smoke + the driver-form bench (20 timed periods after 5 warm-up)
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench20.json 2> gpurun_out/bench20.err
tail -3 gpurun_out/gpu_tests.log; tail -1 gpurun_out/smoke.log; cut -c1-600 gpurun_out/bench20.json

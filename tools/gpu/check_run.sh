# GPU tests and a full-size bench through the VPIC_CHECK build (device bounds traps)
export VPIC_LIB=$PWD/paper_conf_sc_tanlta25_b200/libvpic_check.so
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/check_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/check_tests.log
timeout 600 python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/check_bench.json 2> gpurun_out/check_bench.err; echo "bench rc=$?"
timeout 900 python bench.py --config 2 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/check_bench_c3.json 2> gpurun_out/check_bench_c3.err; echo "bench c3 rc=$?"
tail -2 gpurun_out/check_tests.log; cut -c1-200 gpurun_out/check_bench.json

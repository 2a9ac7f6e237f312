# Round-2 final-build evidence on one B200: GPU tests, smoke, the driver-form bench,
# the launch list of one bench period (ncu, serialised, cold cache: SHARES),
# ncu --set full of k_advance_tma (ions step 0, electrons step 0 and 19) and of
# the sort's fused record pass.
mkdir -p gpurun_out/fin
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/fin/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/fin/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/fin/smoke.log 2>&1
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/fin/bench20.json 2> gpurun_out/fin/bench20.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/fin/launches.csv \
  python bench.py --steps 2 --warmup 1 --profile > gpurun_out/fin/prof_bench.log 2>&1
for sk in 41 40 78; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_advance_tma --launch-skip $sk -c 1 \
  -o gpurun_out/fin/adv_skip$sk python bench.py --steps 1 --warmup 1 --profile > gpurun_out/fin/ncu_adv_$sk.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_radix_pass --launch-skip 2 -c 3 \
  -o gpurun_out/fin/sort_passes python bench.py --steps 1 --warmup 1 --profile > gpurun_out/fin/ncu_sort.log 2>&1
tail -2 gpurun_out/fin/gpu_tests.log; tail -1 gpurun_out/fin/smoke.log; cut -c1-300 gpurun_out/fin/bench20.json
ls -la gpurun_out/fin

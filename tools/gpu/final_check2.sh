# Final evidence for the round (after the interpolator split): kernel mutation test,
# GPU suite, smoke, the driver-form bench, the reference arm, the launch list, ncu
# of k_advance_tma (ions step 0, electrons step 0 and 19).
mkdir -p gpurun_out/final2
timeout 3000 python tools/kernel_mutations.py run --out gpurun_out/final2/kernel_mutations.txt > gpurun_out/final2/mut_run.log 2>&1
rm -f paper_conf_sc_tanlta25_b200/libvpic_mut*.so
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/final2/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/final2/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/final2/smoke.log 2>&1
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/final2/bench20.json 2> gpurun_out/final2/bench20.err
timeout 900 python bench.py --impl reference --gpus 1 --steps 2 --warmup 3 > gpurun_out/final2/bench_ref.json 2> gpurun_out/final2/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final2/launches.csv \
  python bench.py --steps 2 --warmup 1 --profile > gpurun_out/final2/prof_bench.log 2>&1
for sk in 41 40 78; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_advance_tma --launch-skip $sk -c 1 \
  -o gpurun_out/final2/adv_skip$sk python bench.py --steps 1 --warmup 1 --profile > gpurun_out/final2/ncu_adv_$sk.log 2>&1
done
head -2 gpurun_out/final2/kernel_mutations.txt; tail -2 gpurun_out/final2/gpu_tests.log; tail -1 gpurun_out/final2/smoke.log
cut -c1-300 gpurun_out/final2/bench20.json; cut -c1-200 gpurun_out/final2/bench_ref.json

# ncu --set full (with source) of k_advance_tma: electrons at step 0 and step 10 after a sort
for sk in 40 60; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_advance_tma --launch-skip $sk -c 1 \
  -o gpurun_out/adv_el_skip$sk python bench.py --steps 1 --warmup 1 --profile --no-cpu-baseline --no-e2e > gpurun_out/ncu_el_$sk.log 2>&1
tail -2 gpurun_out/ncu_el_$sk.log
done
ls -la gpurun_out/*.ncu-rep

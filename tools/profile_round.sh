set -x
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01_launches.csv python bench.py --steps 2 --warmup 1 --profile > gpurun_out/prof_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_advance_tma --launch-skip 41 -c 1 -o gpurun_out/adv_ion_step0 python bench.py --steps 1 --warmup 1 --profile > gpurun_out/prof1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_advance_tma --launch-skip 78 -c 1 -o gpurun_out/adv_el_step19 python bench.py --steps 1 --warmup 1 --profile > gpurun_out/prof2.log 2>&1
ls -la gpurun_out

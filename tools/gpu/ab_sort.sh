timeout 900 python -m pytest tests/ -x -q -m gpu -k "sort" > gpurun_out/tests_sort.log 2>&1; tail -1 gpurun_out/tests_sort.log
bash tools/gpu/ab.sh "sortold new" 2
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_new.csv python bench.py --steps 1 --warmup 1 --profile > gpurun_out/prof_bench.log 2>&1
python tools/launches.py gpurun_out/launches_new.csv | head -20

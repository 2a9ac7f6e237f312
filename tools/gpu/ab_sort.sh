timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "sort" > gpurun_out/parity_sort.log 2>&1; tail -1 gpurun_out/parity_sort.log
timeout 900 python -m pytest tests/ -x -q -m gpu -k "sort" > gpurun_out/tests_sort.log 2>&1; tail -1 gpurun_out/tests_sort.log
bash tools/gpu/ab.sh "sortold new rilp4" 2

timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "advance or ghost_fill or unload" > gpurun_out/parity_split.log 2>&1; tail -1 gpurun_out/parity_split.log
bash tools/gpu/ab.sh "nosplit new" 3

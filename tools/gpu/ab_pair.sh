timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "advance" > gpurun_out/parity_pair.log 2>&1; tail -1 gpurun_out/parity_pair.log
bash tools/gpu/ab.sh "pr0 new" 3

timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "advance" > gpurun_out/parity_adv.log 2>&1; tail -1 gpurun_out/parity_adv.log
bash tools/gpu/ab.sh "prev new" 3

timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "keyed or sort_parity" > gpurun_out/parity_ck.log 2>&1; tail -1 gpurun_out/parity_ck.log
bash tools/gpu/ab.sh "ck1 new ck8" 2

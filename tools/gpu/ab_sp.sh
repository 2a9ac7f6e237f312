timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "advance" 2>&1 | tail -2
bash tools/gpu/ab.sh "sp0 new" 3

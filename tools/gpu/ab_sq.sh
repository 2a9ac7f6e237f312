VPIC_LIB=$PWD/paper_conf_sc_tanlta25_b200/libvpic_sq.so timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "advance and smem" > gpurun_out/parity_sq.log 2>&1; tail -1 gpurun_out/parity_sq.log
bash tools/gpu/ab.sh "new sq" 3

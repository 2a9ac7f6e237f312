timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "runs_wrap or one_cta or advance_ieee or advance_fast" > gpurun_out/runs_wrap.log 2>&1; tail -2 gpurun_out/runs_wrap.log
timeout 900 python tools/kernel_mutations.py run --only 14 > gpurun_out/mut14.log 2>&1; tail -3 gpurun_out/mut14.log
bash tools/gpu/ab.sh "new" 1

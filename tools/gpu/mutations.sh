timeout 3300 python tools/kernel_mutations.py run --out gpurun_out/kernel_mutations.txt > gpurun_out/mut_run.log 2>&1
tail -3 gpurun_out/mut_run.log
timeout 600 python tools/graph_ab.py --periods 3 > gpurun_out/graph_ab.log 2>&1; tail -6 gpurun_out/graph_ab.log

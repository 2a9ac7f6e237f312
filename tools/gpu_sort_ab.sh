# Dev A/B of radix-pass variants (libvpic_<name>.so): sort parity, sort time
mkdir -p gpurun_out
for n in ${VARIANTS:-base}; do
  if [ "$n" = base ]; then L=""; else L=$PWD/paper_conf_sc_tanlta25_b200/libvpic_$n.so; fi
  VPIC_LIB=$L timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "sort" > gpurun_out/ab_tests_$n.log 2>&1; echo "$n tests rc=$? $(tail -1 gpurun_out/ab_tests_$n.log)"
  for r in 1 2; do VPIC_LIB=$L timeout 300 python tools/sort_bench.py --reps 3 > gpurun_out/ab_sort_$n.log 2>&1; echo "$n $(tail -1 gpurun_out/ab_sort_$n.log)"; done
done

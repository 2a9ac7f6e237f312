# ncu --set full of the radix passes of the first LATE sort of a bench run (after 20 PIC
# steps: launches 6-11 = electrons' three passes, ions' three passes) and the keyed histogram
mkdir -p gpurun_out/sortlate
timeout 900 ncu --set full --clock-control none -k regex:k_radix_pass --launch-skip 6 -c 6 \
  -o gpurun_out/sortlate/passes python bench.py --steps 1 --warmup 1 --profile > gpurun_out/sortlate/ncu1.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:k_count_keys -c 2 \
  -o gpurun_out/sortlate/count python bench.py --steps 1 --warmup 1 --profile > gpurun_out/sortlate/ncu2.log 2>&1
ls gpurun_out/sortlate

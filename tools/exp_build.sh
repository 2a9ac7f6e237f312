#!/bin/bash
# Dev A/B: build libvpic_<name>.so with extra nvcc flags on the FAST advance
# unit (e.g. -DVPIC_EXP=1).  Run with VPIC_LIB=$PWD/paper_conf_sc_tanlta25_b200/libvpic_<name>.so
set -e
name=$1; shift
cd "$(dirname "$0")/.."
B=paper_conf_sc_tanlta25_b200
python -m $B._build >/dev/null
NCCL=$(python -c "import nvidia.nccl,os;print(list(nvidia.nccl.__path__)[0])")
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr \
  -DVPIC_IEEE=0 -fmad=true "$@" -I $NCCL/include -I include -c $B/csrc/advance_p.cu -o /tmp/adv_$name.o
objs=$(ls $B/build/*.o | grep -v advance_fast)
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o $B/libvpic_$name.so /tmp/adv_$name.o $objs \
  -L $NCCL/lib -l:libnccl.so.2 -Xlinker -rpath,$NCCL/lib
echo $B/libvpic_$name.so

#!/bin/bash
# Dev: libvpic_check.so -- the product sources with VPIC_CHECK=1 (device-side
# bounds traps on the hot paths' indices: vpic_internal.cuh VPIC_ASSERT), for
# the GPU parity tests and a full-size bench run through VPIC_LIB.
set -e
cd "$(dirname "$0")/.."
B=paper_conf_sc_tanlta25_b200
python -m $B._build >/dev/null
NCCL=$(python -c "import nvidia.nccl,os;print(list(nvidia.nccl.__path__)[0])")
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr -I $NCCL/include -I include -DVPIC_CHECK=1"
T=$(mktemp -d)
nvcc $F -DVPIC_IEEE=0 -fmad=true -c $B/csrc/advance_p.cu -o $T/advance_fast.o &
nvcc $F -DVPIC_IEEE=1 -fmad=false -prec-div=true -prec-sqrt=true -c $B/csrc/advance_p.cu -o $T/advance_ieee.o &
nvcc $F -c $B/csrc/sort.cu -o $T/sort.o &
wait
objs="$T/advance_fast.o $T/advance_ieee.o $T/sort.o $(ls $B/build/*.o | grep -v -e advance_fast -e advance_ieee -e /sort.o)"
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o $B/libvpic_check.so $objs \
  -L $NCCL/lib -l:libnccl.so.2 -Xlinker -rpath,$NCCL/lib
rm -rf $T
echo $B/libvpic_check.so

#!/bin/bash
# Dev A/B: build libvpic_<name>.so with extra nvcc flags on one unit
# (UNIT=advance (default, FAST advance_p) or UNIT=sort), e.g.
#   ./tools/exp_build.sh nodep -DVPIC_EXP=1
#   UNIT=sort ./tools/exp_build.sh ipt8 -DVPIC_SORT_IPT=8
# Run with VPIC_LIB=$PWD/paper_conf_sc_tanlta25_b200/libvpic_<name>.so
set -e
name=$1; shift
cd "$(dirname "$0")/.."
B=paper_conf_sc_tanlta25_b200
python -m $B._build >/dev/null
NCCL=$(python -c "import nvidia.nccl,os;print(list(nvidia.nccl.__path__)[0])")
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr -I $NCCL/include -I include"
if [ "${UNIT:-advance}" = sort ]; then
  nvcc $F "$@" -c $B/csrc/sort.cu -o /tmp/exp_$name.o
  objs=$(ls $B/build/*.o | grep -v "/sort.o")
else
  nvcc $F -DVPIC_IEEE=0 -fmad=true "$@" -c $B/csrc/advance_p.cu -o /tmp/exp_$name.o
  objs=$(ls $B/build/*.o | grep -v advance_fast)
fi
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o $B/libvpic_$name.so /tmp/exp_$name.o $objs \
  -L $NCCL/lib -l:libnccl.so.2 -Xlinker -rpath,$NCCL/lib
echo $B/libvpic_$name.so

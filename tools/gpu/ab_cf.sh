bash tools/gpu/ab.sh "base new s8 s24 a32s0" 2

bash tools/gpu/ab.sh "new s5a3 s4a1 s5a2" 2

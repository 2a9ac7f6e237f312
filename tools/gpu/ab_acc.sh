bash tools/gpu/ab.sh "new accsoa" 3

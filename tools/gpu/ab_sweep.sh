bash tools/gpu/ab.sh "new cf16 cf32 cf48 ms5 ms10" 2

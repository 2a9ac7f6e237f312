for b in 0 64 128 256 1024; do timeout 600 python tools/group_exp.py --block $b --deposit 2 2>&1 | tail -1; done

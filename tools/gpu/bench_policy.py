"""Dev: bench.py with the AUTO deposit policy's thresholds overridden.
    python tools/gpu/bench_policy.py LO HI [bench args...]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import paper_conf_sc_tanlta25_b200.pic as pic  # noqa: E402

pic.SMEM_SIGMA, pic.SMEM_SIGMA_MAX = float(sys.argv[1]), float(sys.argv[2])
sys.argv = [os.path.join(ROOT, "bench.py")] + sys.argv[3:]
import bench  # noqa: E402

bench.main()

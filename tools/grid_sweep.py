"""Fig. 9 analogue: particle pushes per
nanosecond vs grid size with sorting disabled, total particle count fixed,
push time only.  Particles are in random (shuffled) order, so the cost of
the gather and scatter is set by whether interpolator + accumulator
(144 B per voxel) fit in B200's 126 MB L2.

    python tools/grid_sweep.py [--particles N] [--steps K] > profiles/..jsonl
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_tanlta25_b200 import inputs, vpic  # noqa: E402
from paper_conf_sc_tanlta25_b200.pic import HotPath  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--particles", type=int, default=1 << 27)
    ap.add_argument("--steps", type=int, default=6)
    ap.add_argument("--sizes", default="8,12,16,24,32,40,48,64,80,96,112,128,160,192,256")
    ap.add_argument("--order", default="random", choices=["random", "sorted"])
    args = ap.parse_args()
    for n in [int(x) for x in args.sizes.split(",")]:
        g = inputs.GridSpec(n, n, n)
        ppc = max(1, args.particles // g.ncells)
        wl = inputs.Workload(f"sweep{n}", g, [inputs.Species("electron", -1.0, 1.0, 0.1)], ppc, args.steps, 0)
        p = inputs.particles_in_cells(inputs.uniform_cells(g, ppc), wl.species[0], inputs.MASTER_SEED, 0, 1.0 / ppc)
        if args.order == "random":
            p = inputs.shuffle(p, 5)
        f = inputs.make_fields(g, 0.01)
        hp = HotPath(wl, [p], f, order=vpic.VPIC_SORT_NONE)
        hp.step()
        torch.cuda.synchronize()
        hp.record_advance = True
        hp.adv_events = []
        for _ in range(args.steps):
            hp.step()
        torch.cuda.synchronize()
        ms = sorted(a.elapsed_time(b) for a, b, _ in hp.adv_events)
        med = ms[len(ms) // 2]
        print(json.dumps({"cells": n ** 3, "grid": [n, n, n], "voxels": g.nv, "particles": int(p.size),
                          "ppc": ppc, "order": args.order, "advance_ms_median": med,
                          "pushes_per_ns": p.size / (med * 1e6),
                          "grid_bytes_interp_acc": g.nv * (96 + 48)}), flush=True)
        hp.close()
        del hp
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()

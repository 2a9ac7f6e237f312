"""Dev: time vpic_sort_particles on the C2 electrons after 20 PIC steps (the
disorder the bench's sort sees).  VPIC_LIB selects the library build.
    python tools/sort_bench.py [--steps 20] [--reps 3] [--order standard]"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_tanlta25_b200 import inputs, vpic  # noqa: E402
from paper_conf_sc_tanlta25_b200.pic import HotPath  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--order", default="standard")
ap.add_argument("--config", type=int, default=1)
a = ap.parse_args()
order = {"standard": 0, "strided": 1, "tiled_strided": 2}[a.order]
wl = inputs.config(a.config)
parts = inputs.make_species_particles(wl)
hp = HotPath(wl, parts, inputs.make_fields(wl.grid, wl.field_amp), order=order)
for _ in range(a.steps):
    hp.step()
torch.cuda.synchronize()
res = {}
for k, s in enumerate(hp.species):
    src = s.p.clone()
    ts = []
    for r in range(a.reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        vpic.vpic_sort_particles(hp.ctx, src, s.scratch, s.np, order, 0, hp.ws)
        e1.record()
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    res[s.name] = round(sorted(ts)[len(ts) // 2], 3)
print(json.dumps({"lib": os.environ.get("VPIC_LIB", "default"), "order": a.order, "sort_ms": res}))

"""Dev A/B of advance_p deposit modes on a C2-like uniform plasma (one
species, voxel-sorted, then S PIC steps without re-sorting): per-launch
k_advance time by steps since the sort.

  python tools/adv_ab.py --n 64 --ppc 128 --steps 20 --deposit lane warp
"""
import argparse
import sys
import time

sys.path.insert(0, ".")
import numpy as np
import torch

from paper_conf_sc_tanlta25_b200 import inputs, vpic
from paper_conf_sc_tanlta25_b200.pic import HotPath

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=64)
ap.add_argument("--ppc", type=int, default=128)
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--species", default="electron", choices=["electron", "ion", "both"])
ap.add_argument("--uth", type=float, default=0.0, help="override the electrons' thermal speed")
ap.add_argument("--deposit", nargs="+", default=["warp"])
ap.add_argument("--sigma", type=float, nargs="*", default=[], help="AUTO policy thresholds to try")
a = ap.parse_args()
DEP = {"auto": 0, "lane": 1, "warp": 2, "smem": 3}

wl = inputs.config(1)
from dataclasses import replace
wl = replace(wl, grid=inputs.GridSpec(a.n, a.n, a.n), ppc=a.ppc)
sel = {"electron": [0], "ion": [1], "both": [0, 1]}[a.species]
if a.uth > 0:
    wl = replace(wl, species=[replace(wl.species[0], u_th=a.uth)] + wl.species[1:])
wl = replace(wl, species=[wl.species[k] for k in sel])
t0 = time.time()
parts = inputs.make_species_particles(wl, inputs.MASTER_SEED + 1)
fields = inputs.make_fields(wl.grid, wl.field_amp, inputs.MASTER_SEED + 1)
print(f"# {a.n}^3 x {a.ppc} ppc, {sum(p.size for p in parts)} particles, gen {time.time() - t0:.1f} s",
      flush=True)
import paper_conf_sc_tanlta25_b200.pic as pic
runs = [(d, None) for d in a.deposit] + [("auto", sg) for sg in a.sigma]
for d, sg in runs:
    if sg is not None:
        pic.SMEM_SIGMA = sg
    hp = HotPath(wl, parts, fields, deposit=DEP[d])
    hp.sort()
    hp.record_advance = True
    hp.adv_events = []
    for s in range(a.steps):
        hp.step()
    torch.cuda.synchronize()
    t = [s.elapsed_time(e) for s, e, _ in hp.adv_events]
    jf = hp.jf.sum().item()
    print(d if sg is None else f"auto(sigma={sg})", "mean %.3f ms" % np.mean(t), "by step", [round(x, 3) for x in t[::max(1, len(t) // 10)]],
          "sum(jf) %.6g" % jf, flush=True)
    hp.close()

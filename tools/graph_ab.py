"""Dev A/B: C2 sort periods timed eagerly vs replayed as CUDA graphs
(HotPath(graphs=True)), no per-launch events in either.

  python tools/graph_ab.py [--periods 3]
"""
import argparse
import sys

sys.path.insert(0, ".")
import torch

from paper_conf_sc_tanlta25_b200 import inputs
from paper_conf_sc_tanlta25_b200.pic import HotPath

ap = argparse.ArgumentParser()
ap.add_argument("--periods", type=int, default=3)
ap.add_argument("--config", type=int, default=1)
ap.add_argument("--loopback", action="store_true",
                help="every periodic face through the single-round device-initiated exchange")
a = ap.parse_args()
wl = inputs.config(a.config)
parts = inputs.make_species_particles(wl, inputs.MASTER_SEED + 1)
fields = inputs.make_fields(wl.grid, wl.field_amp, inputs.MASTER_SEED + 1, kind=wl.kind)
S = wl.sort_every
for graphs in (False, True, False, True):
    kw = dict(loopback_exchange=True, device_exchange=True, single_round=True) if a.loopback else {}
    hp = HotPath(wl, parts, fields, graphs=graphs, **kw)
    for _ in range(2):
        hp.cycle(S)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(a.periods):
        hp.cycle(S)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.periods
    hp.sync_counts()
    print(f"loopback={a.loopback} graphs={graphs} {ms:.2f} ms per period, {S * hp.n_particles / ms / 1e6:.2f} G pushes/s", flush=True)
    hp.close()
    del hp
    torch.cuda.empty_cache()

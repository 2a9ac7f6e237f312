"""Upper bound of grouping the records of each B-record block by voxel before
every push (dev experiment): C2, one sort period, the
advance_p launch times by step since the sort with the particle array
re-grouped between steps by torch (untimed) vs untouched.

    python tools/group_exp.py --block 128
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_tanlta25_b200 import inputs  # noqa: E402
from paper_conf_sc_tanlta25_b200.pic import HotPath  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--block", type=int, default=0)
ap.add_argument("--deposit", type=int, default=0)
ap.add_argument("--hash", type=int, default=0, help="group by voxel & (hash-1) instead of voxel")
ap.add_argument("--resort", action="store_true", help="full standard sort before every step (untimed)")
a = ap.parse_args()
wl = inputs.config(1)
parts = inputs.make_species_particles(wl)
hp = HotPath(wl, parts, inputs.make_fields(wl.grid, wl.field_amp), deposit=a.deposit)


def regroup():
    B = a.block
    for s in hp.species:
        n = s.np // B * B
        p = s.p[:n].view(-1, B, 8)
        key = p[..., 3].contiguous().view(torch.int32)
        if a.hash:
            key = key & (a.hash - 1)
        idx = torch.sort(key, dim=1, stable=True).indices
        p.copy_(torch.gather(p, 1, idx.unsqueeze(-1).expand(-1, -1, 8)))


for rep in range(2):
    hp.record_advance = rep == 1
    hp.adv_events = []
    for k in range(20):
        if k and a.block:
            regroup()
        hp.step(do_sort=(k == 0 or a.resort))
    torch.cuda.synchronize()
ms = [e0.elapsed_time(e1) for e0, e1, _ in hp.adv_events]
el, io = ms[0::2], ms[1::2]
print(json.dumps({"resort": a.resort, "block": a.block, "hash": a.hash, "deposit": a.deposit, "mean": round(sum(ms) / len(ms), 3),
                  "electron": [round(x, 2) for x in el], "ion": [round(x, 2) for x in io]}))

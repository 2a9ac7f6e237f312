"""Dev: moving the 32-B records of a late (20 steps after a sort) C2
electron sort by gather (out = in[perm], the product's k_gather) vs scatter
(out[inv] = in, inv = perm^-1) -- torch index kernels for both, ours for
reference.  python tools/gather_vs_scatter.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_tanlta25_b200 import inputs, vpic  # noqa: E402
from paper_conf_sc_tanlta25_b200.pic import HotPath  # noqa: E402

wl = inputs.config(1)
parts = inputs.make_species_particles(wl)
hp = HotPath(wl, parts, inputs.make_fields(wl.grid, wl.field_amp))
for _ in range(20):
    hp.step()
torch.cuda.synchronize()
s = hp.species[0]
n = s.np
src = s.p[:n].clone()
perm = torch.empty(n, dtype=torch.int64, device="cuda")
vpic.vpic_sort_particles(hp.ctx, src, s.scratch, n, 0, 0, hp.ws, None, None, perm)
torch.cuda.synchronize()
inv = torch.empty_like(perm)
inv[perm] = torch.arange(n, device="cuda")
v4 = src.view(-1, 2, 4).view(torch.float32).reshape(n, 8)
out = torch.empty_like(v4)


def t(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


import ctypes
mb = ctypes.CDLL(os.path.join(ROOT, "tools", "mb_scatter.so"))
P = lambda x: ctypes.c_void_p(x.data_ptr())
print("mb gather ms", t(lambda: mb.mb_gather(P(src), P(out), P(perm), ctypes.c_int64(n))))
for v, name in enumerate(["ldg", "nc.L2::64B", "nc.L1::no_allocate", "nc.L2::128B", "cg"]):
    print("mb gather", name, "ms", t(lambda: mb.mb_gatherv(v, P(src), P(out), P(perm), ctypes.c_int64(n))))
print("mb scatter ms", t(lambda: mb.mb_scatter(P(src), P(out), P(inv), ctypes.c_int64(n))))
print("mb invert ms", t(lambda: mb.mb_invert(P(perm), P(inv), ctypes.c_int64(n))))
print("ours (sort incl. gather) ms", t(lambda: vpic.vpic_sort_particles(hp.ctx, src, s.scratch, n, 0, 0, hp.ws)))
print("torch gather out = in[perm] ms", t(lambda: torch.index_select(v4, 0, perm, out=out)))
print("torch scatter out[inv] = in ms", t(lambda: out.index_copy_(0, inv, v4)))
print("torch invert inv[perm] = arange ms", t(lambda: inv.index_copy_(0, perm, torch.arange(n, device='cuda'))))
perm_sorted_sources = torch.arange(n, device="cuda")
print("torch gather identity (coalesced) ms", t(lambda: torch.index_select(v4, 0, perm_sorted_sources, out=out)))

"""Dev: the sort's record gather in an L2-friendly row order vs k_gather
(tools/exp/gather_order.cu).  python tools/exp/gather_order.py"""
import ctypes
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sc_tanlta25_b200 import inputs, vpic  # noqa: E402
from paper_conf_sc_tanlta25_b200.pic import HotPath  # noqa: E402

so = "/tmp/gather_order.so"
subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared", "-Xcompiler",
                       "-fPIC", os.path.join(ROOT, "tools/exp/gather_order.cu"), "-o", so])
lib = ctypes.CDLL(so)
wl = inputs.config(1)
parts = inputs.make_species_particles(wl)
hp = HotPath(wl, parts, inputs.make_fields(wl.grid, wl.field_amp))
for _ in range(20):
    hp.step()
torch.cuda.synchronize()
g = wl.grid
for k, s in enumerate(hp.species):
    n = s.np
    src = s.p[:n].clone()
    perm = torch.empty(n, dtype=torch.int64, device="cuda")
    counts = torch.empty(g.nv, dtype=torch.int32, device="cuda")
    out0 = s.scratch[:n]
    vpic.vpic_sort_particles(hp.ctx, src, out0, n, 0, 0, hp.ws, counts, None, perm)
    torch.cuda.synchronize()
    ref = out0.clone()

    def t(f, reps=5):
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); f(); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        return sorted(ts)[len(ts) // 2]
    ws2 = torch.empty_like(hp.ws)
    sortms = t(lambda: vpic.vpic_sort_particles(hp.ctx, src, out0, n, 0, 0, ws2))
    print(s.name, "full sort (k_gather inside) ms", round(sortms, 3))
    scratch = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    for YB in (2, 4, 8, 16, 130):
        for C in (1024, 4096):
            lib.gather_prep(ctypes.c_void_p(counts.data_ptr()), g.nx + 2, g.ny + 2, g.nz + 2, YB, C,
                            ctypes.c_void_p(scratch.data_ptr()), st)
            torch.cuda.synchronize()
            for blocks in (148 * 4, 148 * 8):
                out = torch.empty_like(src)
                f = lambda: lib.gather_run(ctypes.c_void_p(src.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                           ctypes.c_void_p(perm.data_ptr()), g.nx + 2, g.ny + 2, g.nz + 2, C,
                                           ctypes.c_void_p(scratch.data_ptr()), blocks, st)
                ms = t(f)
                ok = torch.equal(out, ref)
                print(s.name, f"YB={YB} C={C} blocks={blocks}", round(ms, 3), "ms", "ok" if ok else "MISMATCH")

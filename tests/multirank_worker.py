"""Worker of tests/test_gpu_multirank.py (one process per GPU, launched by
torch.distributed.run): the global box split over the ranks, every exchange
mode of csrc/migrate.cu run for real between GPUs (NCCL send/recv or
device-initiated NVLink stores), the results gathered to rank 0 on the
global voxel indices and saved for the test to compare with the oracle.

    python -m torch.distributed.run --nproc-per-node N tests/multirank_worker.py OUT.npz
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sc_tanlta25_b200 import inputs, vpic  # noqa: E402
from paper_conf_sc_tanlta25_b200.pic import HotPath  # noqa: E402

MODES = [("nccl", "rounds"), ("nccl", "single"), ("device", "rounds"), ("device", "single")]


def global_workload():
    """A small uniform box with hot species (many rank crossings) and
    reflecting z walls; split along x (and y, z at 4 / 8 ranks)."""
    gg = inputs.GridSpec(16, 8, 8, dt=0.5, pbc=(0, 0, 1, 0, 0, 1))
    wl = inputs.Workload("multirank", gg, [inputs.Species("electron", -1.0, 1.0, 0.6),
                                           inputs.Species("ion", 1.0, 4.0, 0.3)], 24, 3, 0)
    return wl


def main():
    out = sys.argv[1]
    modes = MODES
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("MR_ONE_GPU") == "1":
        # every rank on GPU 0: NCCL refuses two ranks of one communicator on
        # one device of one host, so each rank poses as its own host
        # (NCCL_HOSTID) and the ranks talk through NCCL's socket transport on
        # the loopback interface -- the real multi-rank NCCL send/recv code
        # path of migrate.cu, without NVLink (so without the device-initiated
        # modes, whose symmetric-memory peers must be NVLink-reachable)
        local = 0
        os.environ["NCCL_HOSTID"] = f"vpic-mr-{rank}"
        os.environ.setdefault("NCCL_SOCKET_IFNAME", "lo")
        os.environ.setdefault("NCCL_IB_DISABLE", "1")
        modes = [m for m in MODES if m[0] == "nccl"]
    torch.cuda.set_device(local)
    dist.init_process_group("gloo" if os.environ.get("MR_ONE_GPU") == "1" else "nccl")
    wl = global_workload()
    gg = wl.grid
    gb = inputs.strong_decompose(gg, world, rank)
    parts = [inputs.to_block(gg, gb, p) for p in inputs.make_species_particles(wl)]
    fields = inputs.block_fields(gg, gb, inputs.make_fields(gg, 0.05))
    from dataclasses import replace
    wlb = replace(wl, grid=gb)
    vb, vg = inputs.block_interior_to_global(gg, gb)
    res = {}
    for exch, mig in modes:
        obj = [vpic.vpic_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        hp = HotPath(wlb, parts, fields, math=vpic.MATH_IEEE, rank=rank, nranks=world, uid=obj[0],
                     device=local, capacity_factor=2.0, device_exchange=exch == "device",
                     inbox_cap=1 << 14, single_round=mig == "single")
        for _ in range(wl.steps):
            hp.step()
        torch.cuda.synchronize()
        mine = {"p%d" % k: inputs.to_global(gg, gb, hp.particles_host(k)) for k in range(len(parts))}
        mine["jf_v"] = vg
        mine["jf"] = hp.jf.cpu().numpy()[vb]
        allr = [None] * world
        dist.all_gather_object(allr, mine)
        if rank == 0:
            for k in range(len(parts)):
                res[f"{exch}_{mig}_p{k}"] = np.concatenate([a["p%d" % k] for a in allr])
            jf = np.zeros((gg.nv, 4), np.float32)
            for a in allr:
                jf[a["jf_v"]] = a["jf"]
            res[f"{exch}_{mig}_jf"] = jf
        hp.close()
        del hp
        dist.barrier()
    if rank == 0:
        np.savez(out, **res)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()

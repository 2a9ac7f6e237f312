"""World-size-2 gloo test of the multi-GPU host logic (CPU, runs here).

The NCCL exchange in csrc/migrate.cu cannot run without GPUs; this test
drives the same protocol, step for step, with torch.distributed (gloo)
between two processes, each advancing its half of a periodic box with the
oracle:

* decomposition (inputs.decompose): process grid 2x1x1, neighbour ranks;
* E/cB halo: plane 1 -> the -face neighbour's plane n+1, axis by axis;
* particle migration: movers classified by exit face (p.i = 8 voxel + face),
  packed with the receiver's entry voxel and flipped offset, counts then
  48-B records exchanged with sends posted in face order and receives in
  opposite-face order (the NCCL matching rule), arrivals appended and their
  move finished, up to 3 rounds;
* jf shared planes: plane n+1 -> +neighbour's plane 1 (added), then plane 1
  -> -neighbour's plane n+1.

The union of both ranks must equal the single-domain oracle: particles
bit-exact (as a multiset in global coordinates), accumulators and jf within
the T1 tolerance.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_tanlta25_b200 import inputs

OPP = [3, 4, 5, 0, 1, 2]
MOVER = np.dtype([("dispx", "<f4"), ("dispy", "<f4"), ("dispz", "<f4"), ("idx", "<i4")])
NG = (8, 6, 5)          # global cells
BLOCK = (4, 6, 5)       # per rank (2x1x1 process grid)
Q, M = -1.0, 1.0


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def global_inputs():
    g = inputs.GridSpec(*NG, dt=0.5)
    p = inputs.random_particles(g, 6000, 77, u_scale=1.2)
    f = inputs.make_fields(g, 0.1, seed=5)
    return g, p, f


def to_local(gg, gl, x0, p):
    """Global voxel -> local voxel for particles inside the block at x0."""
    x, y, z = gg.coords(p["i"])
    q = p.copy()
    q["i"] = gl.voxel(x - x0, y, z)
    return q


def to_global(gg, gl, x0, p):
    x, y, z = gl.coords(p["i"])
    q = p.copy()
    q["i"] = gg.voxel(x + x0, y, z)
    return q


def exchange(recs_by_face, g, kinds, rank):
    """NCCL-order p2p exchange of per-face payloads (float32 [n, 12])."""
    counts = {f: torch.tensor([len(recs_by_face[f])], dtype=torch.int64) for f in range(6)}
    reqs = []
    for f in range(6):
        if kinds[f] == "remote":
            reqs.append(dist.isend(counts[f], g.nbr_rank[f]))
    rc = {}
    for f in range(6):
        o = OPP[f]
        if kinds[o] == "remote":
            rc[o] = torch.zeros(1, dtype=torch.int64)
            reqs.append(dist.irecv(rc[o], g.nbr_rank[o]))
    for r in reqs:
        r.wait()
    reqs = []
    for f in range(6):
        if kinds[f] == "remote" and len(recs_by_face[f]):
            reqs.append(dist.isend(torch.from_numpy(np.ascontiguousarray(recs_by_face[f])), g.nbr_rank[f]))
    bufs = {}
    for f in range(6):
        o = OPP[f]
        if kinds[o] == "remote" and int(rc[o]) > 0:
            bufs[o] = torch.zeros((int(rc[o]), 12), dtype=torch.float32)
            reqs.append(dist.irecv(bufs[o], g.nbr_rank[o]))
    for r in reqs:
        r.wait()
    return [bufs[f].numpy() for f in range(6) if f in bufs]


def worker(rank, world, port, out):
    import oracle
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        gg, pg, fg = global_inputs()
        gl = inputs.decompose(inputs.GridSpec(*BLOCK, dt=0.5), world, rank)
        x0 = gl.gx0
        kinds = ["remote" if gl.nbr_rank[f] != rank else "local" for f in range(6)]
        # ---- fields: interior from the global array, +x ghost plane by halo
        F = fg.reshape(NG[2] + 2, NG[1] + 2, NG[0] + 2, 8)
        fl = np.zeros((gl.nz + 2, gl.ny + 2, gl.nx + 2, 8), np.float32)
        fl[:, :, 1:gl.nx + 1] = F[:, :, x0 + 1:x0 + gl.nx + 1]
        # y, z wrap locally (periodic, 1-wide process grid there): oracle fills
        # them; x: send plane 1 to -x neighbour, receive plane n+1 from +x
        send = torch.from_numpy(np.ascontiguousarray(fl[:, :, 1]))
        recv = torch.zeros_like(send)
        reqs = [dist.isend(send, gl.nbr_rank[0]), dist.irecv(recv, gl.nbr_rank[3])]
        for r in reqs:
            r.wait()
        fl[:, :, gl.nx + 1] = recv.numpy()
        fl = fl.reshape(-1, 8)
        interp = oracle.load_interpolator(gl, fl)
        # ---- particles of this block
        x, _, _ = gg.coords(pg["i"])
        mine = (x - 1 >= x0) & (x - 1 < x0 + gl.nx)
        p = to_local(gg, gl, x0, pg[mine])
        acc = np.zeros((gl.nv, 12), np.float32)
        aabs = np.zeros((gl.nv, 12), np.float64)
        movers = oracle.advance_p(gl, Q, M, p, interp, acc, aabs)
        parts = p
        for rnd in range(3):
            recs = {f: [] for f in range(6)}
            holes = []
            for m in movers:
                i = int(m["idx"])
                code = int(parts["i"][i])
                face, v = code & 7, code >> 3
                holes.append(i)
                if kinds[face] != "remote":
                    continue  # absorbed (none here)
                xx, yy, zz = gl.coords(v)
                q = parts[i].copy()
                a = face % 3
                plus = face >= 3
                if a == 0:
                    xx = 1 if plus else gl.nx
                    q["dx"] = -q["dx"]
                elif a == 1:
                    yy = 1 if plus else gl.ny
                    q["dy"] = -q["dy"]
                else:
                    zz = 1 if plus else gl.nz
                    q["dz"] = -q["dz"]
                q["i"] = gl.voxel(xx, yy, zz)
                rec = np.zeros(12, np.float32)
                rec[:8] = np.frombuffer(q.tobytes(), np.float32)
                rec[8:11] = [m["dispx"], m["dispy"], m["dispz"]]
                recs[face].append(rec)
            recs = {f: (np.array(r, np.float32) if r else np.zeros((0, 12), np.float32)) for f, r in recs.items()}
            arrivals = exchange(recs, gl, kinds, rank)
            keep = np.ones(parts.size, bool)
            keep[holes] = False
            parts = parts[keep]
            movers = []
            for buf in arrivals:
                for rec in buf:
                    q = np.frombuffer(rec[:8].tobytes(), inputs.PARTICLE_DTYPE).copy()
                    mv = np.zeros(1, MOVER)
                    mv["dispx"], mv["dispy"], mv["dispz"] = rec[8], rec[9], rec[10]
                    stop = oracle.move_p(gl, q, mv, acc, Q, aabs)
                    parts = np.concatenate([parts, q])
                    if stop:
                        mv["idx"] = parts.size - 1
                        movers.append(mv[0])
            movers = np.array(movers, MOVER) if movers else np.zeros(0, MOVER)
        assert movers.size == 0
        # ---- jf: unload (y,z folded locally), then the x shared planes
        jf = oracle.unload_accumulator(gl, acc).reshape(gl.nz + 2, gl.ny + 2, gl.nx + 2, 4)
        hi = torch.from_numpy(np.ascontiguousarray(jf[:, :, gl.nx + 1]))
        lo = torch.zeros_like(hi)
        for r in [dist.isend(hi, gl.nbr_rank[3]), dist.irecv(lo, gl.nbr_rank[0])]:
            r.wait()
        jf[:, :, 1] += lo.numpy()
        p1 = torch.from_numpy(np.ascontiguousarray(jf[:, :, 1]))
        gh = torch.zeros_like(p1)
        for r in [dist.isend(p1, gl.nbr_rank[0]), dist.irecv(gh, gl.nbr_rank[3])]:
            r.wait()
        jf[:, :, gl.nx + 1] = gh.numpy()
        out[rank] = dict(p=to_global(gg, gl, x0, parts), acc=acc, aabs=aabs, jf=jf, x0=x0)
    finally:
        dist.destroy_process_group()


def _run(rank, world, port, q):
    out = {}
    worker(rank, world, port, out)
    q.put((rank, out[rank]))


def test_two_rank_step_equals_single_domain(orc):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_run, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=300) for _ in range(2))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    # single-domain reference
    gg, pg, fg = global_inputs()
    interp = orc.load_interpolator(gg, fg.copy())
    p = pg.copy()
    acc = np.zeros((gg.nv, 12), np.float32)
    aabs = np.zeros((gg.nv, 12), np.float64)
    mv = orc.advance_p(gg, Q, M, p, interp, acc, aabs)
    assert mv.size == 0
    # particles: multiset, bit-exact
    both = np.concatenate([res[0]["p"], res[1]["p"]])
    key = lambda a: np.sort(np.ascontiguousarray(a).view(np.dtype((np.void, 32))).ravel())
    assert both.size == p.size
    assert np.array_equal(key(both), key(p))
    # accumulators: each rank's interior voxels map to distinct global voxels
    A = acc.reshape(NG[2] + 2, NG[1] + 2, NG[0] + 2, 12)
    AB = aabs.reshape(A.shape)
    for r in range(2):
        x0 = res[r]["x0"]
        la = res[r]["acc"].reshape(NG[2] + 2, NG[1] + 2, BLOCK[0] + 2, 12)[:, :, 1:BLOCK[0] + 1]
        ga = A[:, :, x0 + 1:x0 + BLOCK[0] + 1]
        gab = AB[:, :, x0 + 1:x0 + BLOCK[0] + 1]
        assert np.all(np.abs(la.astype(np.float64) - ga) <= 1e-5 * gab + 1e-30)
    # jf after the shared-plane reduction equals the global periodic unload
    J = orc.unload_accumulator(gg, acc).reshape(NG[2] + 2, NG[1] + 2, NG[0] + 2, 4)
    Jabs = orc.unload_accumulator(gg, np.abs(acc)).reshape(J.shape).astype(np.float64)
    for r in range(2):
        x0 = res[r]["x0"]
        lj = res[r]["jf"][1:NG[2] + 2, 1:NG[1] + 2, 1:BLOCK[0] + 2]
        gj = J[1:NG[2] + 2, 1:NG[1] + 2, x0 + 1:x0 + BLOCK[0] + 2]
        gjabs = Jabs[1:NG[2] + 2, 1:NG[1] + 2, x0 + 1:x0 + BLOCK[0] + 2]
        assert np.all(np.abs(lj.astype(np.float64) - gj) <= 1e-5 * gjabs + 1e-30), r


def test_decompose_neighbours():
    b = inputs.GridSpec(4, 4, 4)
    for n, grid in ((1, (1, 1, 1)), (2, (2, 1, 1)), (4, (2, 2, 1)), (8, (2, 2, 2))):
        assert inputs.process_grid(n) == grid
        for r in range(n):
            g = inputs.decompose(b, n, r)
            for f in range(6):
                # my neighbour across f sees me across the opposite face
                nb = inputs.decompose(b, n, g.nbr_rank[f])
                assert nb.nbr_rank[OPP[f]] == r
            if n == 1:
                assert g.nbr_rank == (0,) * 6

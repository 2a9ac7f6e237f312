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



def test_strong_decompose_lpi_slab():
    """Strong scaling of configs[4] (bench.py --config 4 at N > 1): the box is
    split over the process grid, and the ranks' slab cells and laser fields
    reassemble exactly the undecomposed box's (slab x in [G/4, 3G/4))."""
    box = inputs.GridSpec(32, 8, 8)
    ref = set()
    for v in inputs.lpi_cells(box, 1):
        x, y, z = box.coords(v)
        ref.add((int(x), int(y), int(z)))
    fref = inputs.make_fields(box, 0.0, kind="lpi")
    for n in (2, 4, 8):
        got = []
        for r in range(n):
            g = inputs.strong_decompose(box, n, r)
            assert (g.gnx, g.nx * inputs.process_grid(n)[0]) == (32, 32)
            for v in inputs.lpi_cells(g, 1):
                x, y, z = g.coords(v)
                assert 1 <= x <= g.nx
                got.append((int(x) + g.gx0, int(y) + g.gy0, int(z) + g.gz0))
            # laser phase follows the global x of every interior voxel
            f = inputs.make_fields(g, 0.0, kind="lpi")
            for v in g.interior_voxels()[:: max(1, g.ncells // 50)]:
                x, y, z = g.coords(v)
                gv = box.voxel(x + g.gx0, y + g.gy0, z + g.gz0)
                assert f[v, 1] == fref[gv, 1] and f[v, 6] == fref[gv, 6]
        assert len(got) == len(set(got)) and set(got) == ref, n
    with pytest.raises(ValueError):
        inputs.strong_decompose(inputs.GridSpec(5, 4, 4), 2, 0)

# ------------------------------------------------ single-round migration --
# Host logic of VPIC_OPT_SINGLE_ROUND_MIGRATION (csrc/migrate.cu:
# ghost_migration_enable, migrate_ghost, reduce_acc_ghosts), replayed with
# gloo between 8 processes on a 2x2x2 process grid -- every direction's
# neighbour is some rank, and along each axis the - and + neighbours coincide,
# the hardest case for pairing sends with receives.
SB = (3, 2, 2)      # block per rank


def compose26(tabs, rank, kinds):
    """Rank of the direction-d neighbour: follow the face neighbours along x,
    then y, then z (the C++ composition); -1 where a crossed face is not
    remote or d is the centre."""
    out = []
    for d in range(27):
        o = (d % 3 - 1, (d // 3) % 3 - 1, d // 9 - 1)
        r, ok = rank, d != 13
        for a in range(3):
            if o[a] == 0 or not ok:
                continue
            f = a if o[a] < 0 else a + 3
            if kinds[f] != "remote":
                ok = False
            else:
                r = tabs[r][f]
        out.append(r if ok else -1)
    return out


def _single_round_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        gl = inputs.decompose(inputs.GridSpec(*SB), world, rank)
        kinds = ["remote" if gl.nbr_rank[f] != rank else "local" for f in range(6)]
        tabs = [None] * world
        dist.all_gather_object(tabs, list(gl.nbr_rank))
        nbr = compose26(tabs, rank, kinds)
        P = inputs.process_grid(world)
        me = (rank % P[0], (rank // P[0]) % P[1], rank // (P[0] * P[1]))
        # 1. the composed rank is the geometric neighbour
        for d in range(27):
            if d == 13:
                continue
            o = (d % 3 - 1, (d // 3) % 3 - 1, d // 9 - 1)
            cc = [(me[a] + o[a]) % P[a] for a in range(3)]
            assert nbr[d] == cc[0] + P[0] * (cc[1] + P[1] * cc[2]), (rank, d)
        # 2. one exchange: per direction a count then records naming (sender,
        #    direction, k); sends in increasing d, receives in decreasing
        #    arrival direction a (= the sender's increasing d)
        cnt = {d: (rank * 27 + d) % 4 for d in range(27) if nbr[d] >= 0}
        reqs = [dist.isend(torch.tensor([cnt[d]], dtype=torch.int64), nbr[d]) for d in sorted(cnt)]
        rc = {}
        for a in range(26, -1, -1):
            if nbr[a] >= 0:
                rc[a] = torch.zeros(1, dtype=torch.int64)
                reqs.append(dist.irecv(rc[a], nbr[a]))
        for r in reqs:
            r.wait()
        reqs = []
        for d in sorted(cnt):
            if cnt[d]:
                rec = torch.tensor([[rank, d, k] for k in range(cnt[d])], dtype=torch.int64)
                reqs.append(dist.isend(rec, nbr[d]))
        got = {}
        for a in range(26, -1, -1):
            if nbr[a] >= 0 and int(rc[a]) > 0:
                got[a] = torch.zeros((int(rc[a]), 3), dtype=torch.int64)
                reqs.append(dist.irecv(got[a], nbr[a]))
        for r in reqs:
            r.wait()
        for a, buf in got.items():
            b = buf.numpy()
            assert np.all(b[:, 0] == nbr[a]) and np.all(b[:, 1] == 26 - a), (rank, a, b)
            assert np.array_equal(b[:, 2], np.arange(len(b)))
        # 3. accumulator ghost layer, axis by axis: plane 0 -> -face neighbour's
        #    plane n, plane n+1 -> +face neighbour's plane 1; receives from +
        #    then -; ghosts zeroed.  Integer-valued float64: sums are exact.
        n = (gl.nx, gl.ny, gl.nz)
        acc = np.zeros((gl.nz + 2, gl.ny + 2, gl.nx + 2, 12))
        rng = np.random.default_rng(100 + rank)
        ghost = np.ones(acc.shape[:3], bool)
        ghost[1:-1, 1:-1, 1:-1] = False
        acc[ghost] = rng.integers(1, 1000, size=(int(ghost.sum()), 12))
        acc[~ghost] = rng.integers(0, 1000, size=(int((~ghost).sum()), 12))
        init = acc.copy()
        for axis in range(3):
            fm, fp = axis, axis + 3
            ax = 2 - axis                                  # numpy axis (z, y, x)
            sl = lambda i: tuple(i if k == ax else slice(None) for k in range(3))
            s0 = torch.from_numpy(acc[sl(0)].copy())
            s1 = torch.from_numpy(acc[sl(n[axis] + 1)].copy())
            acc[sl(0)] = 0
            acc[sl(n[axis] + 1)] = 0
            r2, r3 = torch.zeros_like(s0), torch.zeros_like(s1)
            reqs = [dist.isend(s0, gl.nbr_rank[fm]), dist.isend(s1, gl.nbr_rank[fp]),
                    dist.irecv(r2, gl.nbr_rank[fp]), dist.irecv(r3, gl.nbr_rank[fm])]
            for r in reqs:
                r.wait()
            acc[sl(n[axis])] += r2.numpy()
            acc[sl(1)] += r3.numpy()
        q.put((rank, dict(init=init, acc=acc, gx0=(gl.gx0, gl.gy0, gl.gz0))))
    finally:
        dist.destroy_process_group()


def test_single_round_protocol_eight_ranks():
    """26-neighbour composition, one-exchange pairing, and the axis-ordered
    accumulator ghost reduction: afterwards every ghost value has been added
    to the interior voxel of the rank owning that global voxel (periodic box),
    exactly once, and the ghost layers are zero."""
    world = 8
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_single_round_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    P = inputs.process_grid(world)
    G = (SB[0] * P[0], SB[1] * P[1], SB[2] * P[2])
    want = np.zeros((G[2], G[1], G[0], 12))
    for r in range(world):
        x0, y0, z0 = res[r]["gx0"]
        init = res[r]["init"]
        for z in range(SB[2] + 2):
            for y in range(SB[1] + 2):
                for x in range(SB[0] + 2):
                    want[(z0 + z - 1) % G[2], (y0 + y - 1) % G[1], (x0 + x - 1) % G[0]] += init[z, y, x]
    for r in range(world):
        x0, y0, z0 = res[r]["gx0"]
        acc = res[r]["acc"]
        ghost = np.ones(acc.shape[:3], bool)
        ghost[1:-1, 1:-1, 1:-1] = False
        assert np.all(acc[ghost] == 0)
        got = acc[1:-1, 1:-1, 1:-1]
        assert np.array_equal(got, want[z0:z0 + SB[2], y0:y0 + SB[1], x0:x0 + SB[0]]), r


@pytest.mark.parametrize("nranks", [2, 4, 8])
def test_block_split_roundtrip(nranks):
    """The block views the multi-GPU parity test uses (tests/multirank_worker.py):
    splitting a global box's particles / fields over the process grid and
    mapping them back recovers every particle exactly once and every
    interior field value."""
    from paper_conf_sc_tanlta25_b200 import inputs
    gg = inputs.GridSpec(16, 8, 8, dt=0.5)
    wl = inputs.Workload("split", gg, [inputs.Species("electron", -1.0, 1.0, 0.6)], 5, 1, 0)
    p = inputs.make_species_particles(wl)[0]
    f = inputs.make_fields(gg, 0.05)
    back, cover = [], np.zeros(gg.nv, int)
    for r in range(nranks):
        gb = inputs.strong_decompose(gg, nranks, r)
        pb = inputs.to_block(gg, gb, p)
        back.append(inputs.to_global(gg, gb, pb))
        fb = inputs.block_fields(gg, gb, f)
        vb, vg = inputs.block_interior_to_global(gg, gb)
        assert np.array_equal(fb[vb], f[vg])
        # every block voxel, ghosts included, holds the global value at its
        # global coordinates (outer-face ghost planes are the box's own)
        x, y, z = gb.coords(np.arange(gb.nv))
        assert np.array_equal(fb, f[gg.voxel(x + gb.gx0, y + gb.gy0, z + gb.gz0)])
        cover[vg] += 1
    key = lambda a: np.sort(np.ascontiguousarray(a).view(np.dtype((np.void, 32))))
    assert np.array_equal(key(np.concatenate(back)), key(p))
    assert np.array_equal(cover[gg.interior_voxels()], np.ones(gg.ncells, int))

"""GPU parity of the field solver (vpic_advance_b / vpic_advance_e, §8(f) f1)
and of a self-consistent PIC step (push -> unload -> field advance).

The Yee updates use the oracle's expressions in the same order without FMA,
so fields are bit-exact given identical inputs; through a full step the only
difference is jf (float atomics reordered), bounded by T1.
"""
import numpy as np
import pytest
import torch

from paper_conf_sc_tanlta25_b200 import inputs
from parity_util import assert_particles_bitexact

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def V():
    from paper_conf_sc_tanlta25_b200 import _build, vpic
    _build.build()
    vpic.load()
    return vpic


GRIDS = [inputs.GridSpec(9, 6, 5, dx=0.7, dy=1.0, dz=1.3, dt=0.4),
         inputs.GridSpec(16, 16, 16),
         inputs.GridSpec(7, 5, 4, pbc=(0, 0, 1, 0, 0, 1))]


@pytest.mark.parametrize("g", GRIDS, ids=["noncubic", "cube16", "reflect_z"])
def test_advance_b_e_bitexact(V, orc, g):
    rng = np.random.default_rng(4)
    f = rng.standard_normal((g.nv, 8)).astype(np.float32)
    f[:, 3] = 0
    f[:, 7] = 0
    jf = rng.standard_normal((g.nv, 4)).astype(np.float32)
    ctx = V.Context(g)
    fd = torch.from_numpy(f.copy()).cuda()
    jd = torch.from_numpy(jf).cuda()
    fo = f.copy()
    for frac in (0.5, 0.25, 1.0):
        V.vpic_advance_b(ctx, fd, frac)
        orc.advance_b(g, fo, frac)
        V.vpic_advance_e(ctx, fd, jd, 1.3)
        orc.advance_e(g, fo, jf, 1.3)
    torch.cuda.synchronize()
    got = fd.cpu().numpy()
    assert np.array_equal(got.view(np.uint32), fo.view(np.uint32))


def test_pic_step_with_field_solve(V, orc):
    """Two self-consistent steps (IEEE math): after step 1 the particles are
    bit-exact and the fields within the jf tolerance; step 2 pushes with those
    fields and stays within the FAST-mode tolerances."""
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    wl = inputs.config(0)
    g = wl.grid
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, 0.05)
    hp = HotPath(wl, parts, fields, math=V.MATH_IEEE, field_solve=True)
    hp.step(do_sort=False)
    torch.cuda.synchronize()
    # oracle step
    fo = fields.copy()
    interp = orc.load_interpolator(g, fo)
    acc = np.zeros((g.nv, 12), np.float32)
    aabs = np.zeros((g.nv, 12), np.float64)
    po = [p.copy() for p in parts]
    for sp, p in zip(wl.species, po):
        orc.advance_p(g, sp.q, sp.m, p, interp, acc, aabs)
    jf = orc.unload_accumulator(g, acc)
    jfabs = orc.unload_accumulator(g, np.abs(acc)).astype(np.float64)
    orc.advance_b(g, fo, 0.5)
    orc.advance_e(g, fo, jf, 1.0)
    orc.advance_b(g, fo, 0.5)
    for k in range(2):
        assert_particles_bitexact(hp.particles_host(k), po[k])
    got = hp.fields.cpu().numpy().astype(np.float64)
    cj = g.dt / 1.0
    # E carries -cj * jf (jf within 1e-5 of its abs-sum); cB sees it through curl E
    tol = 1e-5 * cj * jfabs.max() * 4 + 1e-6 * np.abs(fo).max()
    vox = g.interior_voxels()
    assert np.abs(got[vox] - fo[vox].astype(np.float64)).max() <= tol


def _multiset(a):
    return np.sort(np.ascontiguousarray(a).view(np.dtype((np.void, 32))).ravel())


def oracle_steps(orc, g, wl, parts, fields, steps, field_solve=False, eps0=1.0):
    """The single-domain oracle run of `steps` PIC steps (locally periodic
    faces, walls as in g; absorbed particles removed by back-fill): returns
    the particles per species, the last step's jf and its per-edge sum of
    |contributions| (the T1 weights of jf)."""
    po = [p.copy() for p in parts]
    fo = fields.copy()
    for _ in range(steps):
        interp = orc.load_interpolator(g, fo)
        acc = np.zeros((g.nv, 12), np.float32)
        aabs = np.zeros((g.nv, 12), np.float64)
        for k, sp in enumerate(wl.species):
            mv = orc.advance_p(g, sp.q, sp.m, po[k], interp, acc, aabs)
            if mv.size:
                po[k] = orc.remove_absorbed(g, po[k], mv)
        jf = orc.unload_accumulator(g, acc)
        if field_solve:
            orc.advance_b(g, fo, 0.5)
            orc.advance_e(g, fo, jf, eps0)
            orc.advance_b(g, fo, 0.5)
    jf_abs = orc.unload_accumulator(g, aabs.astype(np.float32)).astype(np.float64)
    return po, jf, jf_abs, fo


def assert_jf_t1(g, jf_gpu, jf_orc, jf_abs):
    """T1 on the unloaded currents: per edge |jf_gpu - jf_orc| <= 1e-5 x the
    unloaded sum of |contributions| (periodic fold included)."""
    vox = g.interior_voxels()
    err = np.abs(jf_gpu[vox, :3].astype(np.float64) - jf_orc[vox, :3])
    tol = 1e-5 * jf_abs[vox, :3] + 1e-30
    assert (err <= tol).all(), f"{(err > tol).sum()} jf entries beyond T1, worst {err.max()}"


@pytest.mark.parametrize("walls", [False, True], ids=["periodic", "reflect_z"])
@pytest.mark.parametrize("migration", ["rounds", "single"])
@pytest.mark.parametrize("device_exchange", [False, True], ids=["nccl", "device"])
@pytest.mark.parametrize("field_solve,steps", [(False, 3), (True, 1)])
def test_loopback_exchange_matches_oracle(V, orc, field_solve, steps, device_exchange, migration, walls):
    """VPIC_OPT_LOOPBACK_EXCHANGE sends every periodic crossing, E/cB halo and
    jf shared plane through the NCCL exchange (one-rank communicator, self
    peer): the multi-GPU code path on one GPU.  Compared with the ORACLE's
    single-domain run (IEEE math): particles bit-exact as multisets
    (migration reorders them), jf per edge within T1 of the oracle's, fields
    bit-exact when static (halos move bytes only) and within the jf
    tolerance propagated through the field solve otherwise.  "device":
    the device-initiated exchange (f4) -- the push stores movers into the
    (self) neighbour's symmetric-memory inbox, rounds synchronised on the
    device.  "single": VPIC_OPT_SINGLE_ROUND_MIGRATION -- moves finished in
    the ghost layer, one exchange with the 26 (here: self) neighbours, the
    accumulator's ghost layer added into the boundary voxels; "reflect_z":
    walls on z, so ghost-layer particles also reflect there."""
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    g = inputs.GridSpec(8, 6, 5, dt=0.5, pbc=(0, 0, 1, 0, 0, 1) if walls else (0,) * 6)
    wl = inputs.Workload("loopback", g, [inputs.Species("electron", -1.0, 1.0, 0.6),
                                         inputs.Species("ion", 1.0, 4.0, 0.3)], 40, steps, 0)
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, 0.05)
    runs = []
    for loop in (False, True):
        hp = HotPath(wl, parts, fields, math=V.MATH_IEEE, field_solve=field_solve,
                     loopback_exchange=loop, capacity_factor=1.0,
                     device_exchange=loop and device_exchange, inbox_cap=4096,
                     single_round=loop and migration == "single")
        for _ in range(steps):
            hp.step()
        torch.cuda.synchronize()
        runs.append(hp)
    a, b = runs
    po, jo, jabs, fo = oracle_steps(orc, g, wl, parts, fields, steps, field_solve)
    for k in range(2):
        pa, pb = a.particles_host(k), b.particles_host(k)
        assert pa.size == pb.size == parts[k].size
        assert np.array_equal(_multiset(pb), _multiset(po[k]))    # loopback exchange vs oracle
        assert np.array_equal(_multiset(pa), _multiset(po[k]))    # local wrap vs oracle
        # migration really ran: departed particles were back-filled, arrivals appended
        assert not np.array_equal(pa.view(np.uint32), pb.view(np.uint32))
    assert_jf_t1(g, b.jf.cpu().numpy(), jo, jabs)
    assert_jf_t1(g, a.jf.cpu().numpy(), jo, jabs)
    vox = g.interior_voxels()
    fb = b.fields.cpu().numpy()[vox]
    if not field_solve:
        assert np.array_equal(fb, fo[vox])       # static fields: halos move bytes only
    else:   # E carries -dt/eps0 jf: T1 of jf, carried once through curl E into cB
        tol = 1e-5 * g.dt * jabs.max() * 4 + 1e-6 * np.abs(fo).max()
        assert np.abs(fb.astype(np.float64) - fo[vox]).max() <= tol


@pytest.mark.parametrize("walls", [False, True], ids=["periodic", "absorb_z"])
@pytest.mark.parametrize("migration", ["rounds", "single"])
@pytest.mark.parametrize("device_exchange", [False, True], ids=["nccl", "device"])
def test_loopback_direct_kernel_matches_oracle(V, orc, device_exchange, migration, walls):
    """As above with the direct-load advance kernel (VPIC_OPT_ADVANCE_KERNEL =
    1): its crossers leave through the same move_p / leave() code.  absorb_z:
    absorbing z walls -- particles that enter the ghost layer through x/y and
    then hit a wall there are removed exactly like in the local run."""
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    g = inputs.GridSpec(7, 6, 5, dt=0.5, pbc=(0, 0, 2, 0, 0, 2) if walls else (0,) * 6)
    wl = inputs.Workload("loopback_direct", g, [inputs.Species("electron", -1.0, 1.0, 0.7)], 30, 2, 0)
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, 0.05)
    runs = []
    for loop in (False, True):
        hp = HotPath(wl, parts, fields, math=V.MATH_IEEE, loopback_exchange=loop, capacity_factor=1.0,
                     device_exchange=loop and device_exchange, inbox_cap=4096,
                     single_round=loop and migration == "single")
        hp.ctx.set_option(V.VPIC_OPT_ADVANCE_KERNEL, 1)
        for _ in range(2):
            hp.step()
        torch.cuda.synchronize()
        runs.append(hp)
    a, b = runs
    po, jo, jabs, _ = oracle_steps(orc, g, wl, parts, fields, 2)
    pa, pb = a.particles_host(0), b.particles_host(0)
    if walls:
        assert pa.size < parts[0].size          # some were absorbed
    assert np.array_equal(_multiset(pb), _multiset(po[0]))
    assert np.array_equal(_multiset(pa), _multiset(po[0]))
    assert not np.array_equal(pa.view(np.uint32), pb.view(np.uint32))
    assert_jf_t1(g, b.jf.cpu().numpy(), jo, jabs)
    assert_jf_t1(g, a.jf.cpu().numpy(), jo, jabs)


@pytest.mark.parametrize("migration", ["rounds", "single"])
def test_device_exchange_inbox_overflow_reported(V, migration):
    """An inbox smaller than one round's arrivals: the push keeps going,
    vpic_migrate_particles reports VPIC_ERR_CAPACITY (no silent loss)."""
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    g = inputs.GridSpec(6, 5, 4, dt=0.5)
    wl = inputs.Workload("overflow", g, [inputs.Species("electron", -1.0, 1.0, 0.8)], 60, 1, 0)
    parts = inputs.make_species_particles(wl)
    hp = HotPath(wl, parts, inputs.make_fields(g, 0.05), loopback_exchange=True,
                 device_exchange=True, inbox_cap=2, capacity_factor=1.0,
                 single_round=migration == "single")
    with pytest.raises(V.VpicError) as ei:
        hp.step()
    assert ei.value.status == -2      # VPIC_ERR_CAPACITY


@pytest.mark.timeout(300)
@pytest.mark.parametrize("exchange", ["none", "loopback"])
def test_graph_mode_matches_eager(V, exchange):
    """HotPath(graphs=True): the PIC steps of each sort period captured once per
    particle-buffer configuration (CUDA graph) and replayed, particle counts on
    the device (vpic_advance_p_dev / vpic_migrate_particles_dev).  Three sort
    periods (eager warm-up, capture + replay, replay of the other buffer
    configuration's graph...) must reproduce the eager run: bit-identical
    arrays without exchange, equal multisets with the loopback single-round
    exchange; jf within the reordering tolerance."""
    import gc
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    gc.collect()                        # no other test's context (NCCL communicator) alive
    g = inputs.GridSpec(8, 6, 5, dt=0.5)
    wl = inputs.Workload("graphs", g, [inputs.Species("electron", -1.0, 1.0, 0.6),
                                       inputs.Species("ion", 1.0, 4.0, 0.3)], 40, 4, 4)
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, 0.05)
    loop = exchange == "loopback"
    res = []
    for graphs in (False, True):      # one context (one NCCL communicator) at a time
        hp = HotPath(wl, parts, fields, math=V.MATH_IEEE, loopback_exchange=loop, device_exchange=loop,
                     single_round=loop, inbox_cap=4096, capacity_factor=1.0, graphs=graphs)
        for _ in range(4):
            hp.cycle(4)
        torch.cuda.synchronize()
        res.append(([hp.particles_host(k) for k in range(2)], hp.jf.cpu().numpy(), len(hp._graphs)))
        hp.close()
    (pa, ja, _), (pb, jb, ng) = res
    assert ng == 2                      # one graph per buffer configuration, replayed
    for k in range(2):
        if loop:
            assert np.array_equal(_multiset(pa[k]), _multiset(pb[k]))
        else:
            assert np.array_equal(pa[k].view(np.uint32), pb[k].view(np.uint32))
    vox = g.interior_voxels()
    assert np.abs(ja[vox] - jb[vox]).max() <= 1e-5 * np.abs(ja[vox]).max() * 8


@pytest.mark.parametrize("exchange,migration", [("nccl", "rounds"), ("nccl", "single"),
                                                ("device", "rounds"), ("device", "single")])
def test_mover_list_overflow_refused(V, exchange, migration):
    """advance_p with a mover list smaller than the step's departures: the
    push drops the excess (flags bit 0) and vpic_migrate_particles -- every
    exchange path -- reports VPIC_ERR_CAPACITY instead of reading movers past
    the list (migrate took the count from *n_movers unclamped)."""
    import gc
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    gc.collect()
    g = inputs.GridSpec(6, 5, 4, dt=0.5)
    wl = inputs.Workload("mv_overflow", g, [inputs.Species("electron", -1.0, 1.0, 0.8)], 60, 1, 0)
    parts = inputs.make_species_particles(wl)
    hp = HotPath(wl, parts, inputs.make_fields(g, 0.05), loopback_exchange=True,
                 device_exchange=exchange == "device", inbox_cap=1 << 16, capacity_factor=1.0,
                 single_round=migration == "single", max_movers=8)
    with pytest.raises(V.VpicError) as ei:
        hp.step()
    assert ei.value.status == -2      # VPIC_ERR_CAPACITY
    torch.cuda.synchronize()
    hp.close()

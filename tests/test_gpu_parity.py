"""GPU parity: every C-ABI call against the oracle on identical seeded inputs.

Bars: sort keys, counts, new keys and permutation
bit-exact; interpolator bit-exact; particles bit-exact in IEEE mode and within
4 ulp / 1e-6 (oracle voxel frame) in FAST mode; accumulators and jf within
1e-5 of the sum of absolute contributions (atomic reordering only).
"""
import numpy as np
import pytest
import torch

from paper_conf_sc_tanlta25_b200 import inputs
from parity_util import (assert_acc_close, assert_particles_bitexact, assert_particles_close,
                         kick_bound, replay_inputs, u_of)

pytestmark = pytest.mark.gpu
PD = inputs.PARTICLE_DTYPE


@pytest.fixture(scope="module")
def V():
    from paper_conf_sc_tanlta25_b200 import _build, vpic
    _build.build()
    vpic.load()
    assert torch.cuda.is_available(), "gpu tests need a B200"
    return vpic


def mkctx(V, g, math=0, deposit=0, kernel=0):
    c = V.Context(g)
    c.set_option(V.VPIC_OPT_MATH, math)
    c.set_option(V.VPIC_OPT_DEPOSIT, deposit)
    c.set_option(V.VPIC_OPT_ADVANCE_KERNEL, kernel)
    return c


def dev_particles(V, p):
    return V.particles_to_device(p)


def harris_small():
    """configs[2]'s Harris sheet (sech^2 density, tanh cB_x, reflecting z,
    drifting species) on a 24x8x32 grid, 40 ppc mean: ~4x the background
    density in the sheet -- the contention case."""
    from dataclasses import replace
    wl = inputs.config(2)
    wh = replace(wl, grid=inputs.GridSpec(24, 8, 32, pbc=wl.grid.pbc), ppc=40)
    return wh, inputs.make_species_particles(wh)


def lpi_small():
    """configs[4]'s laser-plasma slab (plasma in x in [nx/4, 3nx/4), hot
    electrons u_th = 0.2 drifting at u_x = +0.3, cold heavy ions, static
    laser ey = cbz = 0.02 sin(2 pi x / 32)) on a 64x8x8 grid, 24 ppc: the
    high-crossing, empty-voxel case."""
    from dataclasses import replace
    wl = inputs.config(4)
    wlp = replace(wl, grid=inputs.GridSpec(64, 8, 8), ppc=24)
    return wlp, inputs.make_species_particles(wlp)


# ------------------------------------------------------------------ sort --
def sort_cases():
    out = []
    wl = inputs.config(0)
    pe = inputs.make_species_particles(wl)[0]
    out.append(("c1_sorted", wl.grid, pe))
    out.append(("c1_shuffled", wl.grid, inputs.shuffle(pe, 1)))
    g = inputs.GridSpec(7, 5, 3)
    out.append(("random_ragged", g, inputs.random_particles(g, 8193, 2)))
    out.append(("three_voxels", g, inputs.random_particles(g, 5000, 3, vox=[g.voxel(1, 1, 1), g.voxel(7, 5, 3), g.voxel(3, 2, 2)])))
    out.append(("one_voxel", g, inputs.random_particles(g, 10000, 4, vox=[g.voxel(4, 3, 2)])))
    out.append(("single", g, inputs.random_particles(g, 1, 5)))
    out.append(("warp_minus_one", g, inputs.random_particles(g, 31, 6)))
    g2 = inputs.GridSpec(32, 32, 32)
    out.append(("many_tiles", g2, inputs.shuffle(inputs.random_particles(g2, 200000, 7), 8)))
    # more radix tiles (407 of 6144, ragged last) than one wave of resident
    # CTAs (with VPIC_SORT_PERSIST each CTA loops over several tickets)
    g3 = inputs.GridSpec(64, 64, 64)
    out.append(("multi_wave", g3, inputs.shuffle(inputs.random_particles(g3, 2500001, 11), 12)))
    wh, ph = harris_small()
    out.append(("harris_sheet", wh.grid, inputs.shuffle(ph[1], 9)))
    return out


@pytest.mark.parametrize("case", sort_cases(), ids=lambda c: c[0])
@pytest.mark.parametrize("order,T", [(0, 0), (1, 0), (2, 7), (2, 1), (2, 0), (3, 0)])
def test_sort_parity(V, orc, case, order, T):
    name, g, p = case
    ctx = mkctx(V, g)
    Tq = T if T else ctx.info()["tile_sz"]
    p_out_o, counts_o, nk_o, perm_o = orc.sort_particles(g, p, order, Tq)
    n = p.size
    p_in = dev_particles(V, p)
    p_out = torch.empty_like(p_in)
    ws = torch.empty(V.vpic_sort_workspace_bytes(ctx, n, order), dtype=torch.uint8, device="cuda")
    counts = torch.full((g.nv,), -7, dtype=torch.int32, device="cuda")
    nk = torch.empty(n, dtype=torch.int64, device="cuda")
    perm = torch.empty(n, dtype=torch.int64, device="cuda")
    V.vpic_sort_particles(ctx, p_in, p_out, n, order, T, ws, counts, nk, perm)
    torch.cuda.synchronize()
    assert_particles_bitexact(V.particles_to_host(p_out), p_out_o)
    assert np.array_equal(counts.cpu().numpy(), counts_o)
    assert np.array_equal(perm.cpu().numpy(), perm_o)
    assert np.array_equal(nk.cpu().numpy(), nk_o)
    # input untouched
    assert_particles_bitexact(V.particles_to_host(p_in), p)


def test_sort_three_passes(V, orc):
    """nv > 2^26: the standard sort needs three <= 13-bit digit passes."""
    g = inputs.GridSpec(512, 512, 256)
    p = inputs.random_particles(g, 100000, 9)
    ctx = mkctx(V, g)
    p_out_o, counts_o, _, perm_o = orc.sort_particles(g, p, 0)
    p_in = dev_particles(V, p)
    p_out = torch.empty_like(p_in)
    ws = torch.empty(V.vpic_sort_workspace_bytes(ctx, p.size, 0), dtype=torch.uint8, device="cuda")
    counts = torch.empty(g.nv, dtype=torch.int32, device="cuda")
    perm = torch.empty(p.size, dtype=torch.int64, device="cuda")
    V.vpic_sort_particles(ctx, p_in, p_out, p.size, 0, 0, ws, counts, None, perm)
    assert np.array_equal(perm.cpu().numpy(), perm_o)
    assert np.array_equal(counts.cpu().numpy(), counts_o)


def test_sort_empty(V):
    g = inputs.GridSpec(4, 4, 4)
    ctx = mkctx(V, g)
    counts = torch.full((g.nv,), 5, dtype=torch.int32, device="cuda")
    x = torch.empty((0, 8), device="cuda")
    for order in range(4):
        V.vpic_sort_particles(ctx, x, torch.empty_like(x), 0, order, 0, None, counts)
        assert int(counts.abs().sum()) == 0


# ----------------------------------------------------- interp / advance --
def adv_cases():
    wl = inputs.config(0)
    ps = inputs.make_species_particles(wl)
    g = wl.grid
    f = inputs.make_fields(g, 0.01)
    out = [("c1_electrons", g, ps[0], -1.0, 1.0, f), ("c1_ions", g, ps[1], 1.0, 25.0, f)]
    gh = inputs.GridSpec(9, 6, 5, pbc=(0, 0, 1, 0, 0, 1))
    out.append(("reflect_z_hot", gh, inputs.random_particles(gh, 20000, 11, u_scale=1.0), -1.0, 1.0,
                inputs.make_fields(gh, 0.05, seed=3)))
    gr = inputs.GridSpec(5, 6, 7)
    out.append(("periodic_hot_ragged", gr, inputs.random_particles(gr, 12345, 12, u_scale=1.2), 0.7,
                1.3, inputs.make_fields(gr, 0.2, seed=4)))
    wh, ph = harris_small()
    out.append(("harris_sheet_electrons", wh.grid, ph[0], -1.0, 1.0,
                inputs.make_fields(wh.grid, 0.01, kind="harris")))
    wp, pp = lpi_small()
    out.append(("lpi_slab_electrons", wp.grid, pp[0], -1.0, 1.0,
                inputs.make_fields(wp.grid, 0.01, kind="lpi")))
    # non-cubic cells (every cdt/d and cell-size factor distinct; dt under the
    # Courant limit of the smallest cell)
    R = inputs.BC_REFLECT
    gn = inputs.GridSpec(8, 7, 6, dx=0.6, dy=1.4, dz=1.0, dt=0.4, pbc=(0, R, 0, 0, R, 0))
    out.append(("noncubic_cells", gn, inputs.random_particles(gn, 15000, 14, u_scale=0.8), -1.0, 1.0,
                inputs.make_fields(gn, 0.05, seed=6)))
    # random order on 40^3 voxels: every warp's items in distinct voxels
    gs = inputs.GridSpec(40, 40, 40)
    out.append(("scattered_cache_overflow", gs, inputs.random_particles(gs, 150000, 13, u_scale=0.5),
                -1.0, 1.0, inputs.make_fields(gs, 0.02, seed=5)))
    # voxel-sorted, ~125 per voxel, with items moved into the x-neighbour voxel
    # where they sit (crossed since the sort): 5% in the first half (chunks of
    # the carry-first deposit, <= 24 stragglers), 40% in the second (chunks of
    # the general segment loop), voxels changing inside chunks
    gq = inputs.GridSpec(8, 8, 8)
    pq = inputs.random_particles(gq, 64000, 15, u_scale=0.3)
    pq = pq[np.argsort(pq["i"], kind="stable")]
    rng = np.random.default_rng(16)
    frac = np.where(np.arange(pq.size) < pq.size // 2, 0.05, 0.40)
    mv = rng.random(pq.size) < frac
    x = pq["i"] % (gq.nx + 2)
    pq["i"] = np.where(mv, pq["i"] + np.where(x < gq.nx, 1, -1), pq["i"])
    out.append(("sorted_stragglers", gq, pq, -1.0, 1.0, inputs.make_fields(gq, 0.02, seed=7)))
    return out



def assert_replay_exact(orc, g, q, p, r):
    """FAST mode: the oracle's move + deposit of the GPU's pushed momenta."""
    pr = replay_inputs(orc, g, q, p, r["p"])
    acc_r = np.zeros((g.nv, 12), np.float32)
    abs_r = np.zeros((g.nv, 12), np.float64)
    mv_r = orc.move_deposit(g, q, pr, acc_r, abs_r)
    assert_particles_bitexact(r["p"], pr)
    assert_acc_close(r["acc"], acc_r, abs_r)
    assert r["nm"] == mv_r.size
    key = lambda m: np.sort(np.ascontiguousarray(m).view(np.dtype((np.void, 16))))
    if mv_r.size:
        mv_gpu = r["movers"][:r["nm"]].copy().view(mv_r.dtype).reshape(-1)
        assert np.array_equal(key(mv_gpu), key(mv_r))


def run_both(V, orc, g, p, q, m, fields, math, deposit, kernel=0):
    interp_o = orc.load_interpolator(g, fields.copy())
    acc_o = np.zeros((g.nv, 12), np.float32)
    acc_abs = np.zeros((g.nv, 12), np.float64)
    acc_cond = np.zeros((g.nv, 12), np.float64)
    p_o = p.copy()
    mv_o = orc.advance_p(g, q, m, p_o, interp_o, acc_o, acc_abs, acc_cond=acc_cond)
    ctx = mkctx(V, g, math, deposit, kernel)
    fd = torch.from_numpy(fields.copy()).cuda()
    interp = torch.zeros((g.nv, 24), dtype=torch.float32, device="cuda")
    V.vpic_load_interpolator(ctx, fd, interp)
    acc = torch.empty((g.nv, 12), dtype=torch.float32, device="cuda")
    V.vpic_clear_accumulator(ctx, acc)
    pd = dev_particles(V, p)
    movers = torch.zeros((max(p.size, 1), 4), dtype=torch.float32, device="cuda")
    nm = torch.zeros(1, dtype=torch.int64, device="cuda")
    flags = torch.zeros(1, dtype=torch.int32, device="cuda")
    V.vpic_advance_p(ctx, q, m, pd, p.size, interp, acc, movers, p.size, nm, flags)
    torch.cuda.synchronize()
    return dict(interp_o=interp_o, acc_o=acc_o, acc_abs=acc_abs, acc_cond=acc_cond, p_o=p_o, mv_o=mv_o,
                interp=interp.cpu().numpy(), acc=acc.cpu().numpy(), p=V.particles_to_host(pd),
                nm=int(nm.item()), flags=int(flags.item()), ctx=ctx, fields=fd.cpu().numpy(),
                acc_t=acc, movers=movers.cpu().numpy())


@pytest.mark.parametrize("case", adv_cases(), ids=lambda c: c[0])
@pytest.mark.parametrize("deposit", [1, 2, 3], ids=["lane", "warp", "smem"])
@pytest.mark.parametrize("kernel", [1, 2], ids=["direct", "tma"])
def test_advance_ieee_bitexact(V, orc, case, deposit, kernel):
    name, g, p, q, m, f = case
    r = run_both(V, orc, g, p, q, m, f, V.MATH_IEEE, deposit, kernel)
    vox = g.interior_voxels()
    coef = V.interp_coefficients(r["interp"], g.nv)
    assert np.array_equal(coef[vox], r["interp_o"][vox, :18])
    assert np.all(r["interp_o"][vox, 18:] == 0)
    assert_particles_bitexact(r["p"], r["p_o"])
    assert_acc_close(r["acc"], r["acc_o"], r["acc_abs"])
    assert r["nm"] == 0 and r["flags"] == 0


@pytest.mark.parametrize("case", adv_cases(), ids=lambda c: c[0])
@pytest.mark.parametrize("deposit", [1, 2, 3], ids=["lane", "warp", "smem"])
@pytest.mark.parametrize("kernel", [1, 2], ids=["direct", "tma"])
def test_advance_fast_tolerance(V, orc, case, deposit, kernel):
    name, g, p, q, m, f = case
    r = run_both(V, orc, g, p, q, m, f, V.MATH_FAST, deposit, kernel)
    # (1) the push: momenta (and positions) within T2 of the oracle's step;
    # T2's kick term is a rare exception, not the working tolerance
    nkick = assert_particles_close(g, r["p"], r["p_o"], u_of(p), kick_bound(g, p, q, m, r["interp_o"]))
    assert nkick <= max(2, p.size // 2000), nkick
    # (2) the move and the deposit are the oracle's exactly, given the pushed
    # momenta (VPIC_EXACT_MOVE): replaying the GPU's momenta through the
    # oracle's move_p + ACCUMULATE_J gives the GPU's particles bit for bit and
    # its accumulator up to summation order (T1)
    assert_replay_exact(orc, g, q, p, r)
    nt3 = int((np.abs(r["acc"].astype(np.float64) - r["acc_o"]) > 1e-5 * r["acc_abs"] + 1e-30).sum())
    print(f"[{name}] T2 kick term: {nkick} of {p.size} particles; entries beyond T1 of the oracle's "
          f"own step (different momenta): {nt3} of {int((r['acc_abs'] > 0).sum())}")


def test_ghost_fill_matches(V, orc):
    g = inputs.GridSpec(6, 5, 4)
    f = inputs.make_fields(g, 1.0, seed=9)
    r = run_both(V, orc, g, inputs.random_particles(g, 10, 1), 1.0, 1.0, f, V.MATH_IEEE, 1)
    fo = f.copy()
    orc.load_interpolator(g, fo)
    assert np.array_equal(r["fields"], fo)


@pytest.mark.parametrize("case", adv_cases()[2:], ids=lambda c: c[0])
def test_unload_parity(V, orc, case):
    name, g, p, q, m, f = case
    r = run_both(V, orc, g, p, q, m, f, V.MATH_FAST, 2)
    jf = torch.empty((g.nv, 4), dtype=torch.float32, device="cuda")
    V.vpic_unload_accumulator(r["ctx"], r["acc_t"], jf)
    jf_o = orc.unload_accumulator(g, r["acc"])
    jf_abs = orc.unload_accumulator(g, np.abs(r["acc"])).astype(np.float64)
    assert_acc_close(jf.cpu().numpy(), jf_o, jf_abs + 1e-30)


def test_continuity_on_gpu_output(V, orc):
    """Discrete continuity 4 dR + div J = 0 evaluated on the GPU's particles and
    accumulator (FAST mode, warp deposit)."""
    g = inputs.GridSpec(8, 8, 8, dt=0.5)
    p = inputs.random_particles(g, 50000, 21, u_scale=0.8)
    q = 0.7
    rho0 = orc.accumulate_rho(g, p, q)
    r = run_both(V, orc, g, p, q, 1.0, inputs.make_fields(g, 0.05), V.MATH_FAST, 2)
    rho1 = orc.accumulate_rho(g, r["p"], q)
    J = orc.unload_raw(g, r["acc"])
    S = (g.nx + 2, g.ny + 2, g.nz + 2)
    Jg = J[:, :3].reshape(S[2], S[1], S[0], 3).transpose(2, 1, 0, 3).copy()
    R = (rho1 - rho0).reshape(S[2], S[1], S[0]).transpose(2, 1, 0).copy()
    for a in range(3):
        hi = [slice(None)] * 3; hi[a] = S[a] - 1
        lo = [slice(None)] * 3; lo[a] = 1
        Jg[tuple(lo)] += Jg[tuple(hi)]
        R[tuple(lo)] += R[tuple(hi)]
    core = (slice(1, S[0] - 1), slice(1, S[1] - 1), slice(1, S[2] - 1))
    res = 4 * R[core]
    for a in range(3):
        Ja = Jg[core + (a,)]
        res = res + Ja - np.roll(Ja, 1, axis=a)
    scale = np.abs(4 * R[core]).max()
    assert scale > 1
    assert np.abs(res).max() < 2e-5 * scale


@pytest.mark.parametrize("kernel", [1, 2], ids=["direct", "tma"])
def test_absorb_movers_and_migrate(V, orc, kernel):
    """Absorbing z walls: movers reported, particles removed (multiset equal
    to the oracle's back-fill; IEEE mode so records are bit-identical)."""
    g = inputs.GridSpec(6, 6, 3, pbc=(0, 0, 2, 0, 0, 2))
    p = inputs.random_particles(g, 9000, 31, u_scale=1.5)
    r = run_both(V, orc, g, p, -1.0, 1.0, inputs.make_fields(g, 0.01), V.MATH_IEEE, 2, kernel)
    assert r["nm"] == r["mv_o"].size > 0
    assert_particles_bitexact(r["p"], r["p_o"])
    # migrate on the GPU
    pd = dev_particles(V, r["p"])
    ctx = r["ctx"]
    # rebuild the mover list on the device from the oracle's (same set)
    movers = torch.from_numpy(r["mv_o"].copy().view(np.float32).reshape(-1, 4)).cuda()
    nm = torch.tensor([r["mv_o"].size], dtype=torch.int64, device="cuda")
    n_new = V.vpic_migrate_particles(ctx, -1.0, 1.0, pd, p.size, p.size, movers, movers.shape[0], nm,
                                     r["acc_t"])
    p_left_o = orc.remove_absorbed(g, r["p_o"].copy(), r["mv_o"])
    assert n_new == p_left_o.size
    got = V.particles_to_host(pd[:n_new])
    key = lambda a: np.sort(np.ascontiguousarray(a).view(np.dtype((np.void, 32))))
    assert np.array_equal(key(got), key(p_left_o))


def test_mover_overflow_flag(V, orc):
    g = inputs.GridSpec(6, 6, 3, pbc=(0, 0, 2, 0, 0, 2))
    p = inputs.random_particles(g, 9000, 31, u_scale=1.5)
    ctx = mkctx(V, g)
    fd = torch.from_numpy(inputs.make_fields(g, 0.01)).cuda()
    interp = torch.zeros((g.nv, 24), device="cuda")
    V.vpic_load_interpolator(ctx, fd, interp)
    acc = torch.zeros((g.nv, 12), device="cuda")
    pd = dev_particles(V, p)
    movers = torch.zeros((4, 4), device="cuda")
    nm = torch.zeros(1, dtype=torch.int64, device="cuda")
    flags = torch.zeros(1, dtype=torch.int32, device="cuda")
    V.vpic_advance_p(ctx, -1.0, 1.0, pd, p.size, interp, acc, movers, 4, nm, flags)
    torch.cuda.synchronize()
    assert int(nm.item()) > 4 and int(flags.item()) & 1
    # the migration refuses the overflowed list before touching anything
    before = V.particles_to_host(pd)
    with pytest.raises(V.VpicError) as ei:
        V.vpic_migrate_particles(ctx, -1.0, 1.0, pd, p.size, p.size, movers, 4, nm, acc)
    assert ei.value.status == V.VPIC_ERR_CAPACITY
    assert_particles_bitexact(V.particles_to_host(pd), before)


def test_invalid_arguments(V):
    g = inputs.GridSpec(4, 4, 4)
    ctx = mkctx(V, g)
    with pytest.raises(V.VpicError):
        ctx.set_option(V.VPIC_OPT_MATH, 7)
    x = torch.zeros((10, 8), device="cuda")
    with pytest.raises(V.VpicError):  # in-place sort is rejected
        V.vpic_sort_particles(ctx, x, x, 10, 0, 0, torch.empty(1 << 20, dtype=torch.uint8, device="cuda"))
    with pytest.raises(V.VpicError):  # workspace too small
        V.vpic_sort_particles(ctx, x, torch.empty_like(x), 10, 0, 0, torch.empty(16, dtype=torch.uint8, device="cuda"))
    with pytest.raises(V.VpicError):
        V.Context(inputs.GridSpec(4, 4, 4, nbr_rank=(1, 0, 0, 0, 0, 0)))


def test_run_host_cycles_matches_device_cycles(V):
    """The pipelined host-streaming driver (e2e path of bench.py) returns the
    same particles as device-resident cycles on the same inputs."""
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    wl = inputs.config(0)
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(wl.grid, wl.field_amp)
    ref = HotPath(wl, parts, fields)
    ref.cycle(4)
    torch.cuda.synchronize()
    want = [ref.particles_host(k) for k in range(2)]
    hp = HotPath(wl, parts, fields)
    host_in = [torch.from_numpy(np.ascontiguousarray(p).view(np.float32).reshape(-1, 8)).pin_memory()
               for p in parts]
    host_out = [torch.empty(tuple(h.shape), dtype=torch.float32, pin_memory=True) for h in host_in]
    jf_host = torch.empty((wl.grid.nv, 4), dtype=torch.float32, pin_memory=True)
    f_host = torch.from_numpy(fields).pin_memory()
    n = hp.run_host_cycles(host_in, host_out, f_host, jf_host, 3, 4)
    torch.cuda.synchronize()
    assert n == 3 * 4 * sum(p.size for p in parts)
    for k in range(2):
        got = host_out[k].numpy().view(inputs.PARTICLE_DTYPE).reshape(-1)
        assert_particles_bitexact(got, want[k])
    assert np.all(np.isfinite(jf_host.numpy()))


@pytest.mark.parametrize("nx", [0, 37])
@pytest.mark.parametrize("agg", [0, 1])
@pytest.mark.parametrize("order", ["sorted", "strided", "random"])
def test_gather_scatter_parity(V, orc, nx, agg, order):
    rng = np.random.default_rng(5)
    K, m = 3001, 70
    if order == "sorted":
        keys = np.repeat(np.arange(K), m)
    elif order == "strided":
        keys = np.tile(np.arange(K), m)
    else:
        keys = rng.permutation(np.repeat(np.arange(K), m))
    keys = keys.astype(np.int32)
    x = rng.standard_normal(keys.size)
    table = rng.standard_normal(K)
    acc_o = np.zeros(K)
    out_o = orc.gather_scatter(keys, x, table, acc_o, nx)
    ctx = mkctx(V, inputs.GridSpec(4, 4, 4))
    kd, xd, td = (torch.from_numpy(a).cuda() for a in (keys, x, table))
    out = torch.empty_like(xd)
    acc = torch.zeros(K, dtype=torch.float64, device="cuda")
    V.vpic_gather_scatter(ctx, kd, xd, td, out, acc, nx, agg)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), out_o)               # same summation order
    absum = np.zeros(K)
    orc.gather_scatter(keys, np.abs(x), table, absum, nx)
    assert np.all(np.abs(acc.cpu().numpy() - acc_o) <= 1e-13 * absum + 1e-300)


# Chunk-schedule edges of k_advance_tma: 64-particle chunks dealt in pairs,
# full chunks through the tensor map, the ragged one through a plain bulk
# copy, the last voxel's sum carried across a pair.  Sorted voxel runs of
# 96 (a voxel straddles chunk and pair boundaries) with hot particles so the
# chunk-closing items are often crossers.
@pytest.mark.parametrize("n", [1, 63, 64, 65, 127, 128, 129, 191, 4097, 70000])
@pytest.mark.parametrize("deposit", [2, 3], ids=["warp", "smem"])
def test_advance_chunk_edges_ieee(V, orc, n, deposit):
    g = inputs.GridSpec(12, 10, 8)
    vox = np.repeat(g.interior_voxels(), 96)[:n]
    p = inputs.random_particles(g, n, 31 + n, u_scale=0.9)
    p["i"] = vox
    r = run_both(V, orc, g, p, -1.0, 1.0, inputs.make_fields(g, 0.05, seed=8), V.MATH_IEEE, deposit, 2)
    assert_particles_bitexact(r["p"], r["p_o"])
    assert_acc_close(r["acc"], r["acc_o"], r["acc_abs"])


# ------------------------------------------ move_p edge cases (reading R13) --
def edge_case_particles(g):
    """Particles built so that move_p meets its degenerate branches, with the
    fields zero (u is unchanged by the push, so the displacements below are
    exact): on a face moving out of it (zero-length first streak), on a face
    moving in, zero displacement on one or two axes (the 3.4e38 branch), exact
    two- and three-face ties (equal offsets and momenta on a cubic grid: the
    lower axis wins, strict '<'), a track ending exactly on a face (in-cell,
    d = +-1 kept), and corner crossings through the periodic wrap."""
    cells = [(x, y, z) for z in (1, 2, g.nz) for y in (1, 2, g.ny) for x in (1, 2, g.nx)]
    rows = []
    u = 0.5
    for s in (+1.0, -1.0):
        rows += [((s, 0.3, -0.2), (s * u, 0.1, 0.0)),          # on +-x face, moving out
                 ((0.2, s, 0.1), (0.0, s * u, -0.2)),          # on +-y face, moving out, ux = 0
                 ((0.1, -0.4, s), (0.0, 0.0, s * u)),          # on +-z face, only z moving
                 ((s, s, 0.0), (s * u, s * u, 0.0)),           # on an edge, moving out of both
                 ((s, s, s), (s * u, s * u, s * u)),           # on a corner, moving out of all
                 ((s, 0.0, 0.0), (-s * u, 0.0, 0.0)),          # on a face, moving in
                 ((0.9 * s, 0.9 * s, 0.0), (s * u, s * u, 0.0)),       # two-face tie x = y
                 ((0.0, 0.9 * s, 0.9 * s), (0.0, s * u, s * u)),       # two-face tie y = z
                 ((0.9 * s, 0.9 * s, 0.9 * s), (s * u, s * u, s * u)),  # three-face tie
                 ((0.7 * s, -0.7 * s, 0.7 * s), (s * u, -s * u, s * u)),  # three-face tie, mixed signs
                 ((0.0, 0.0, 0.0), (0.0, 0.0, 0.0)),                  # at rest: all disp == 0
                 ((0.6 * s, 0.0, 0.0), (2.0 * s, 0.0, 0.0))]          # fast, single axis
    # a track ending exactly on the face: d + 2 disp == 1 in float32
    n = len(rows) * len(cells)
    p = np.zeros(n + len(cells), PD)
    k = 0
    for c in cells:
        for d, uu in rows:
            p[k]["i"] = g.voxel(*c)
            p[k]["dx"], p[k]["dy"], p[k]["dz"] = d
            p[k]["ux"], p[k]["uy"], p[k]["uz"] = uu
            p[k]["w"] = 0.25 + 0.01 * (k % 7)
            k += 1
    # in float32 with VPIC's half displacement (ux c dt / dx) / gamma at ux = 1
    # (c dt / dx = 0.5 below): the offset whose track ends exactly on +x
    f32 = np.float32
    disp = (f32(1.0) * f32(0.5)) * (f32(1.0) / np.sqrt(f32(1.0) + f32(1.0) * f32(1.0)))
    d_end = f32(1.0) - f32(2.0) * disp
    for _ in range(8):
        e = (d_end + disp) + disp
        if e == f32(1.0):
            break
        d_end = np.nextafter(d_end, f32(2.0) if e < 1 else f32(-2.0), dtype=np.float32)
    assert (d_end + disp) + disp == f32(1.0)
    for c in cells:
        p[k]["i"] = g.voxel(*c)
        p[k]["dx"], p[k]["dy"], p[k]["dz"] = d_end, 0.0, 0.0
        p[k]["ux"] = 1.0
        p[k]["w"] = 1.0
        k += 1
    return p


@pytest.mark.parametrize("pbc", [(0,) * 6, (1, 0, 2, 1, 0, 2)], ids=["periodic", "walls"])
@pytest.mark.parametrize("deposit", [1, 2, 3], ids=["lane", "warp", "smem"])
@pytest.mark.parametrize("kernel", [1, 2], ids=["direct", "tma"])
def test_advance_edge_cases_ieee(V, orc, pbc, deposit, kernel):
    g = inputs.GridSpec(5, 5, 5, pbc=pbc, dt=0.5)
    p = edge_case_particles(g)
    f = np.zeros((g.nv, 8), np.float32)
    r = run_both(V, orc, g, p, -1.0, 1.0, f, V.MATH_IEEE, deposit, kernel)
    assert_particles_bitexact(r["p"], r["p_o"])
    assert_acc_close(r["acc"], r["acc_o"], r["acc_abs"])
    assert r["nm"] == r["mv_o"].size
    key = lambda m: np.sort(np.ascontiguousarray(m).view(np.dtype((np.void, 16))))
    if r["nm"]:
        # absorbed movers: the same {remaining displacement, index} set
        mv_gpu = r["movers"][:r["nm"]].copy().view(r["mv_o"].dtype).reshape(-1)
        assert np.array_equal(key(mv_gpu), key(r["mv_o"]))


def test_edge_case_particles_exercise_the_branches(orc):
    """The edge-case set really reaches the branches it names: crossings with
    zero-length first streaks, ties, particles left exactly on faces."""
    g = inputs.GridSpec(5, 5, 5, dt=0.5)
    p = edge_case_particles(g)
    f = np.zeros((g.nv, 8), np.float32)
    interp = orc.load_interpolator(g, f)
    acc = np.zeros((g.nv, 12), np.float32)
    p1 = p.copy()
    orc.advance_p(g, -1.0, 1.0, p1, interp, acc)
    moved = p1["i"] != p["i"]
    assert moved.sum() > p.size // 3
    ended_on_face = p1["dx"][-27:] == 1.0            # the exact end-of-track tie (with 2)
    assert ended_on_face.all() and np.array_equal(p1["i"][-27:], p["i"][-27:])


@pytest.mark.parametrize("order", [0, 1, 2], ids=["standard", "strided", "tiled"])
def test_sort_captures_in_cuda_graph(V, orc, order):
    """Every order is stream-ordered with no host synchronisation (the rank
    passes are sized on the device), so vpic_sort_particles can be captured
    in a CUDA graph; replays on new input bytes stay bit-exact."""
    g = inputs.GridSpec(20, 18, 16)
    ctx = mkctx(V, g)
    T = 37
    n = 60001
    p_in = torch.empty((n, 8), dtype=torch.float32, device="cuda")
    p_out = torch.empty_like(p_in)
    ws = torch.empty(V.vpic_sort_workspace_bytes(ctx, n, order), dtype=torch.uint8, device="cuda")
    counts = torch.empty(g.nv, dtype=torch.int32, device="cuda")
    nk = torch.empty(n, dtype=torch.int64, device="cuda")
    perm = torch.empty(n, dtype=torch.int64, device="cuda")
    p0 = inputs.shuffle(inputs.random_particles(g, n, 71), 72)
    p_in.copy_(V.particles_to_device(p0))
    V.vpic_sort_particles(ctx, p_in, p_out, n, order, T, ws, counts, nk, perm)   # warm-up (attributes)
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    gr = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        with torch.cuda.graph(gr, stream=s):
            V.vpic_sort_particles(ctx, p_in, p_out, n, order, T, ws, counts, nk, perm, stream=s)
    for seed in (73, 74):
        # a different key distribution each replay: max_r, min_k, max_k change
        vox = None if seed == 73 else [g.voxel(3, 4, 5), g.voxel(20, 18, 16), g.voxel(7, 1, 2)]
        p = inputs.shuffle(inputs.random_particles(g, n, seed, vox=vox), seed + 10)
        p_in.copy_(V.particles_to_device(p))
        gr.replay()
        torch.cuda.synchronize()
        p_o, c_o, nk_o, perm_o = orc.sort_particles(g, p, order, T)
        assert_particles_bitexact(V.particles_to_host(p_out), p_o)
        assert np.array_equal(counts.cpu().numpy(), c_o)
        assert np.array_equal(nk.cpu().numpy(), nk_o)
        assert np.array_equal(perm.cpu().numpy(), perm_o)


@pytest.mark.parametrize("order", [0, 1, 2], ids=["standard", "strided", "tiled"])
def test_keyed_sort_matches_sort(V, orc, order):
    """vpic_advance_p_keys writes every particle's voxel after its move (in-cell
    items in the chunk, crossers after the drain); vpic_sort_particles_keyed
    on those keys gives exactly the oracle's sort of the advanced particles
    (hot particles: many crossers; ragged size; both kernels)."""
    g = inputs.GridSpec(12, 9, 7)
    p = inputs.random_particles(g, 40001, 81, u_scale=0.7)
    f = inputs.make_fields(g, 0.05, seed=6)
    for kernel in (1, 2):
        ctx = mkctx(V, g, V.MATH_IEEE, 2, kernel)
        fd = torch.from_numpy(f.copy()).cuda()
        interp = torch.zeros((g.nv, 24), dtype=torch.float32, device="cuda")
        V.vpic_load_interpolator(ctx, fd, interp)
        acc = torch.zeros((g.nv, 12), dtype=torch.float32, device="cuda")
        pd = dev_particles(V, p)
        nm = torch.zeros(1, dtype=torch.int64, device="cuda")
        keys = torch.full((p.size,), -5, dtype=torch.int32, device="cuda")
        V.vpic_advance_p_keys(ctx, -1.0, 1.0, pd, p.size, interp, acc, None, 0, nm, None, keys)
        torch.cuda.synchronize()
        assert int(nm.item()) == 0
        adv = V.particles_to_host(pd)
        assert np.array_equal(keys.cpu().numpy(), adv["i"])
        T = 29
        out = torch.empty_like(pd)
        ws = torch.empty(V.vpic_sort_workspace_bytes(ctx, p.size, order), dtype=torch.uint8, device="cuda")
        counts = torch.empty(g.nv, dtype=torch.int32, device="cuda")
        nk = torch.empty(p.size, dtype=torch.int64, device="cuda")
        perm = torch.empty(p.size, dtype=torch.int64, device="cuda")
        V.vpic_sort_particles_keyed(ctx, pd, out, p.size, order, T, keys, ws, counts, nk, perm)
        torch.cuda.synchronize()
        p_o, c_o, nk_o, perm_o = orc.sort_particles(g, adv, order, T)
        assert_particles_bitexact(V.particles_to_host(out), p_o)
        assert np.array_equal(counts.cpu().numpy(), c_o)
        assert np.array_equal(nk.cpu().numpy(), nk_o)
        assert np.array_equal(perm.cpu().numpy(), perm_o)
        if order == 0:
            # no voxel histogram asked for: digit histograms straight from the keys
            out2 = torch.empty_like(pd)
            perm2 = torch.full((p.size,), -3, dtype=torch.int64, device="cuda")
            V.vpic_sort_particles_keyed(ctx, pd, out2, p.size, order, T, keys, ws, None, None, perm2)
            torch.cuda.synchronize()
            assert_particles_bitexact(V.particles_to_host(out2), p_o)
            assert np.array_equal(perm2.cpu().numpy(), perm_o)
            out3 = torch.empty_like(pd)
            V.vpic_sort_particles_keyed(ctx, pd, out3, p.size, order, T, keys, ws, None, None, None)
            torch.cuda.synchronize()
            assert_particles_bitexact(V.particles_to_host(out3), p_o)


def test_keyed_cycles_match_unkeyed(V):
    """HotPath with the keyed sort (the default) and without: identical
    particles after two sort periods (IEEE math)."""
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    g = inputs.GridSpec(10, 8, 6, dt=0.5)
    wl = inputs.Workload("keyed", g, [inputs.Species("electron", -1.0, 1.0, 0.5),
                                      inputs.Species("ion", 1.0, 9.0, 0.1)], 20, 4, 4)
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, 0.05)
    res = []
    for keyed in (True, False):
        hp = HotPath(wl, parts, fields, math=V.MATH_IEEE, keyed_sort=keyed)
        hp.cycle(4)
        hp.cycle(4)
        torch.cuda.synchronize()
        res.append([hp.particles_host(k) for k in range(2)])
    for k in range(2):
        assert_particles_bitexact(res[0][k], res[1][k])


@pytest.mark.parametrize("deposit", [2, 3], ids=["warp", "smem"])
def test_advance_runs_wrap_bitexact(V, orc, deposit):
    """More chunk runs than warps (1 CTA per SM, 1.6 M voxel-sorted particles:
    > 16 x 8 x 148 chunks), so every warp goes on to later runs (runs of 16
    consecutive chunks in WARP mode, pairs in SMEM mode) and carries its
    voxel across chunks: IEEE particles bit-exact, accumulator within T1."""
    g = inputs.GridSpec(32, 32, 32)
    p = inputs.random_particles(g, 1600000, 91, u_scale=0.3)
    p = p[np.argsort(p["i"], kind="stable")]
    f = inputs.make_fields(g, 0.02, seed=8)
    interp_o = orc.load_interpolator(g, f.copy())
    acc_o = np.zeros((g.nv, 12), np.float32)
    acc_abs = np.zeros((g.nv, 12), np.float64)
    p_o = p.copy()
    orc.advance_p(g, -1.0, 1.0, p_o, interp_o, acc_o, acc_abs)
    ctx = mkctx(V, g, V.MATH_IEEE, deposit, 2)
    ctx.set_option(V.VPIC_OPT_ADVANCE_CTAS_PER_SM, 1)
    assert 64 * 16 * 8 * ctx.info()["num_sms"] < p.size
    fd = torch.from_numpy(f.copy()).cuda()
    interp = torch.zeros((g.nv, 24), dtype=torch.float32, device="cuda")
    V.vpic_load_interpolator(ctx, fd, interp)
    acc = torch.zeros((g.nv, 12), dtype=torch.float32, device="cuda")
    pd = dev_particles(V, p)
    nm = torch.zeros(1, dtype=torch.int64, device="cuda")
    V.vpic_advance_p(ctx, -1.0, 1.0, pd, p.size, interp, acc, None, 0, nm, None)
    torch.cuda.synchronize()
    assert int(nm.item()) == 0
    assert_particles_bitexact(V.particles_to_host(pd), p_o)
    assert_acc_close(acc.cpu().numpy(), acc_o, acc_abs)


def test_advance_one_cta_per_sm_bitexact(V, orc):
    """VPIC_OPT_ADVANCE_CTAS_PER_SM = 1 (half the persistent grid) gives the
    oracle's particles too."""
    wl = inputs.config(0)
    g = wl.grid
    p = inputs.make_species_particles(wl)[0]
    f = inputs.make_fields(g, 0.01)
    interp_o = orc.load_interpolator(g, f.copy())
    acc_o = np.zeros((g.nv, 12), np.float32)
    acc_abs = np.zeros((g.nv, 12), np.float64)
    p_o = p.copy()
    orc.advance_p(g, -1.0, 1.0, p_o, interp_o, acc_o, acc_abs)
    ctx = mkctx(V, g, V.MATH_IEEE, 2, 2)
    ctx.set_option(V.VPIC_OPT_ADVANCE_CTAS_PER_SM, 1)
    fd = torch.from_numpy(f.copy()).cuda()
    interp = torch.zeros((g.nv, 24), dtype=torch.float32, device="cuda")
    V.vpic_load_interpolator(ctx, fd, interp)
    acc = torch.zeros((g.nv, 12), dtype=torch.float32, device="cuda")
    pd = dev_particles(V, p)
    nm = torch.zeros(1, dtype=torch.int64, device="cuda")
    V.vpic_advance_p(ctx, -1.0, 1.0, pd, p.size, interp, acc, None, 0, nm, None)
    torch.cuda.synchronize()
    assert_particles_bitexact(V.particles_to_host(pd), p_o)
    assert_acc_close(acc.cpu().numpy(), acc_o, acc_abs)


def test_sort_tiled_64bit_rank_keys(V, orc):
    """TILED_STRIDED whose rank keys (chunk - chunk0) * max_r + r exceed 32
    bits (T = 1 over a 2^18-voxel key range, 20000 particles in one voxel):
    the 64-bit chain of rank passes runs; bit-exact against the oracle."""
    g = inputs.GridSpec(64, 64, 64)
    lo, hi, mid = g.voxel(1, 1, 1), g.voxel(64, 64, 64), g.voxel(30, 31, 32)
    p = inputs.random_particles(g, 20003, 91, vox=[mid])
    p["i"][:2] = lo
    p["i"][-1] = hi
    p = inputs.shuffle(p, 92)
    assert (hi - lo) * 20000 > 2**32
    ctx = mkctx(V, g)
    n = p.size
    p_in = dev_particles(V, p)
    p_out = torch.empty_like(p_in)
    ws = torch.empty(V.vpic_sort_workspace_bytes(ctx, n, 2), dtype=torch.uint8, device="cuda")
    nk = torch.empty(n, dtype=torch.int64, device="cuda")
    perm = torch.empty(n, dtype=torch.int64, device="cuda")
    V.vpic_sort_particles(ctx, p_in, p_out, n, 2, 1, ws, None, nk, perm)
    torch.cuda.synchronize()
    p_o, _, nk_o, perm_o = orc.sort_particles(g, p, 2, 1)
    assert nk_o.max() >= 2**32
    assert_particles_bitexact(V.particles_to_host(p_out), p_o)
    assert np.array_equal(nk.cpu().numpy(), nk_o)
    assert np.array_equal(perm.cpu().numpy(), perm_o)

"""Pins for the oracle's push / move / deposit (VPIC reading).

Expected values come from physics and geometry, not from the oracle:
* uniform E, B = 0: u_n = u_0 + 2 n qdt_2mc E, bit-exact for dyadic inputs;
  position advances by u c dt / (gamma dx) per step (relativistic velocity);
* uniform B: |u| conserved (the Boris rotation is a rotation); the rotation
  angle per step equals the exact cyclotron angle 2 phi = 2 qdt_2mc |B| / gamma
  up to the O(phi^7) remainder of the 5th-order tan series that the
  tan-corrected Boris uses (reading R11); positive charges turn clockwise
  about B; the orbit is a regular polygon: chord L = |u| c dt / gamma and
  circumradius R = L / (2 sin(theta/2));
* E x B: the guiding centre drifts at E x B / B^2;
* move_p: offsets stay in [-1,1]; the global displacement telescopes to the
  requested one; reflect mirrors; absorb / remote report the exit face;
* charge conservation: 4 (R_new - R_old) + div J = 0 at every node
  (Delta rho + Delta t div J = 0, the discrete continuity invariant);
* deposit totals: sum of all jx partials = 4 sum q disp_x.
"""
import math

import numpy as np
import pytest

from paper_conf_sc_tanlta25_b200 import inputs

PD = inputs.PARTICLE_DTYPE


def grid(n=4, dt=0.5, pbc=(0,) * 6, nbr=(0,) * 6):
    return inputs.GridSpec(n, n, n, dt=dt, pbc=tuple(pbc), nbr_rank=tuple(nbr))


def uniform_fields(g, E=(0, 0, 0), B=(0, 0, 0)):
    f = np.zeros((g.nv, 8), np.float32)
    f[:, 0:3] = np.array(E, np.float32)
    f[:, 4:7] = np.array(B, np.float32)
    return f


def one_particle(g, cell=(2, 2, 2), d=(0, 0, 0), u=(0, 0, 0), w=1.0):
    p = np.zeros(1, PD)
    p["i"] = g.voxel(*cell)
    p["dx"], p["dy"], p["dz"] = d
    p["ux"], p["uy"], p["uz"] = u
    p["w"] = w
    return p


def global_pos(g, p):
    """Physical position in cell units: voxel (x,y,z) spans [x, x+1]."""
    x, y, z = g.coords(p["i"])
    return np.stack([x + (1 + p["dx"].astype(np.float64)) / 2,
                     y + (1 + p["dy"].astype(np.float64)) / 2,
                     z + (1 + p["dz"].astype(np.float64)) / 2], -1)


def unwrap_step(prev, cur, n):
    d = cur - prev
    return d - n * np.round(d / n)


def run(orc, g, p, fields, q, m, steps, track=False):
    interp = orc.load_interpolator(g, fields)
    acc = np.zeros((g.nv, 12), np.float32)
    us, xs = [], []
    pos = global_pos(g, p)
    disp = np.zeros_like(pos)
    for _ in range(steps):
        acc[:] = 0
        mv = orc.advance_p(g, q, m, p, interp, acc)
        assert mv.size == 0
        new = global_pos(g, p)
        disp += unwrap_step(pos, new, np.array([g.nx, g.ny, g.nz]))
        pos = new
        if track:
            us.append(np.array([p["ux"][0], p["uy"][0], p["uz"][0]], np.float64))
            xs.append(disp[0].copy())
    return np.array(us), np.array(xs)


def test_uniform_E_bit_exact(orc):
    """TV1: qdt_2mc = 1/4, E = (2^-8, -2^-9, 2^-7)."""
    g = grid(dt=0.5)
    E = (2.0**-8, -(2.0**-9), 2.0**-7)
    p = one_particle(g)
    us, xs = run(orc, g, p, uniform_fields(g, E=E), 1.0, 1.0, 300, track=True)
    n = np.arange(1, 301)[:, None]
    expect = n * 2 * 0.25 * np.array(E)
    assert np.array_equal(us, expect)  # bit-exact
    # position: sum_n u_n c dt / gamma_n (cells), in double
    gam = np.sqrt(1 + (expect**2).sum(1))[:, None]
    xexp = np.cumsum(expect * 0.5 / gam, 0)
    assert np.abs(xs - xexp).max() < 2e-5
    assert abs(xs[-1, 0]) > 4  # crossed the periodic box more than once


def test_gyration(orc):
    """TV2: qdt_2mc = 0.3, cB = (0,0,1.3), u0 = (0.4,0,0), E = 0."""
    g = grid(dt=0.6)
    p = one_particle(g, u=(0.4, 0.0, 0.0))
    us, xs = run(orc, g, p, uniform_fields(g, B=(0, 0, 1.3)), 1.0, 1.0, 2000, track=True)
    umag = np.linalg.norm(us, axis=1)
    assert np.abs(umag - 0.4).max() < 4e-6          # energy conserved
    assert np.all(us[:, 2] == 0)
    ang = np.arctan2(us[:, 1], us[:, 0])
    dth = np.diff(np.concatenate([[0.0], ang]))
    dth = (dth + np.pi) % (2 * np.pi) - np.pi
    assert np.all(dth < 0)                          # q > 0 turns clockwise about +z
    gamma = math.sqrt(1 + 0.16)
    phi = 0.3 * 1.3 / gamma
    theta = -dth.mean()
    remainder = 2 * (17.0 / 315.0) * phi**7
    assert abs(theta - 2 * phi) < 1.5 * remainder + 1e-6
    assert abs(theta - 2 * phi) > 0.3 * remainder   # the tan correction is truncated, not exact
    # regular polygon: chord and circumradius
    L = 0.4 * 0.6 / gamma
    chords = np.linalg.norm(np.diff(xs[:, :2], axis=0), axis=1)
    assert np.abs(chords - L).max() < 2e-6
    a = xs[:-2, :2]; b = xs[1:-1, :2]; c = xs[2:, :2]
    la = np.linalg.norm(b - c, axis=1); lb = np.linalg.norm(a - c, axis=1); lc = np.linalg.norm(a - b, axis=1)
    area = 0.5 * np.abs((b - a)[:, 0] * (c - a)[:, 1] - (b - a)[:, 1] * (c - a)[:, 0])
    R = np.median(la * lb * lc / (4 * area))
    assert abs(R - L / (2 * math.sin(theta / 2))) / R < 2e-4


def test_ExB_drift(orc):
    """Small phi: the particle started at the drift speed keeps E x B / B^2."""
    g = grid(dt=0.05)
    vd = 0.01
    p = one_particle(g, u=(vd / math.sqrt(1 - vd * vd), 0, 0))
    steps = 4000
    us, xs = run(orc, g, p, uniform_fields(g, E=(0, vd, 0), B=(0, 0, 1.0)), 1.0, 1.0, steps, track=True)
    v = xs[-1] / (steps * 0.05)
    assert abs(v[0] - vd) / vd < 2e-3
    assert abs(v[1]) < 1e-5 and v[2] == 0


def test_ExB_drift_negative_charge(orc):
    g = grid(dt=0.05)
    vd = 0.01
    p = one_particle(g, u=(vd / math.sqrt(1 - vd * vd), 0, 0))
    steps = 4000
    _, xs = run(orc, g, p, uniform_fields(g, E=(0, vd, 0), B=(0, 0, 1.0)), -1.0, 1.0, steps, track=True)
    v = xs[-1] / (steps * 0.05)
    assert abs(v[0] - vd) / vd < 2e-3   # E x B drift is charge independent


def _random_movers(g, n, seed, scale=0.99):
    rng = np.random.default_rng(seed)
    p = inputs.random_particles(g, n, seed)
    disp = (rng.random((n, 3)) * 2 - 1) * scale
    return p, disp.astype(np.float32)


def test_move_p_geometry_periodic(orc):
    g = grid(n=3)
    p, disp = _random_movers(g, 3000, 5)
    # put some particles exactly on faces and give some zero displacement
    p["dx"][:100] = 1.0
    p["dy"][100:200] = -1.0
    disp[200:300, 1] = 0.0
    acc = np.zeros((g.nv, 12), np.float32)
    pos0 = global_pos(g, p)
    for k in range(p.size):
        pk = p[k:k + 1].copy()
        mv = _mover(disp[k])
        assert orc.move_p(g, pk, mv, acc, 1.0) == 0
        assert mv["dispx"][0] == 0 or abs(mv["dispx"][0]) < 1e-6
        p[k] = pk[0]
    assert np.all(np.abs(p["dx"]) <= 1) and np.all(np.abs(p["dy"]) <= 1) and np.all(np.abs(p["dz"]) <= 1)
    x, y, z = g.coords(p["i"])
    assert np.all((x >= 1) & (x <= 3) & (y >= 1) & (y <= 3) & (z >= 1) & (z <= 3))
    moved = unwrap_step(pos0, global_pos(g, p), np.array([3, 3, 3]))
    assert np.abs(moved - disp.astype(np.float64)).max() < 2e-6


def _mover(d):
    mv = np.zeros(1, np.dtype([("dispx", "<f4"), ("dispy", "<f4"), ("dispz", "<f4"), ("idx", "<i4")]))
    mv["dispx"], mv["dispy"], mv["dispz"] = d
    return mv


def test_move_p_reflect_absorb_remote(orc):
    g = grid(n=4, pbc=(0, 0, 1, 0, 0, 2), nbr=(0, 0, 0, 0, 1, 0))
    acc = np.zeros((g.nv, 12), np.float32)
    # reflect at -z: z=1 cell, offset -0.5, moving -z by 0.5 cells (disp 0.5 offset units -> 1.0)
    p = one_particle(g, cell=(2, 2, 1), d=(0, 0, -0.5), u=(0, 0, -0.3))
    X0 = global_pos(g, p)[0]
    assert orc.move_p(g, p, _mover((0.1, 0.0, -0.5)), acc, 1.0) == 0
    X1 = global_pos(g, p)[0]
    assert p["uz"][0] == np.float32(0.3)
    # unreflected z would be X0 - 0.5 = 0.75 - 0.5 = 0.25 -> mirrored about z=1 -> 1.75
    assert abs(X1[2] - (2 * 1.0 - (X0[2] - 0.5))) < 1e-6
    assert abs(X1[0] - (X0[0] + 0.1)) < 1e-6
    # absorb at +z
    p = one_particle(g, cell=(3, 1, 4), d=(0.2, 0, 0.5), u=(0, 0, 0.3))
    mv = _mover((0.0, 0.0, 0.5))
    assert orc.move_p(g, p, mv, acc, 1.0) == 1
    assert p["i"][0] == 8 * g.voxel(3, 1, 4) + 5 and p["dz"][0] == 1.0
    assert abs(mv["dispz"][0] - 0.25) < 1e-7
    # remote at +y (nbr_rank[+y] = 1 != rank 0)
    p = one_particle(g, cell=(1, 4, 2), d=(0, 0.9, 0), u=(0, 0.3, 0))
    mv = _mover((0.0, 0.2, 0.0))
    assert orc.move_p(g, p, mv, acc, 1.0) == 1
    assert p["i"][0] == 8 * g.voxel(1, 4, 2) + 4 and p["dy"][0] == 1.0
    assert abs(mv["dispy"][0] - 0.15) < 1e-7


def _continuity(orc, g, n, seed, fields_amp, q=0.7, perturb=0.0):
    rng = np.random.default_rng(seed)
    p = inputs.random_particles(g, n, seed, u_scale=0.8)
    fields = (rng.random((g.nv, 8)) * 2 - 1).astype(np.float32) * np.float32(fields_amp)
    interp = orc.load_interpolator(g, fields)
    acc = np.zeros((g.nv, 12), np.float32)
    rho0 = orc.accumulate_rho(g, p, q)
    orc.advance_p(g, q, 1.0, p, interp, acc)
    rho1 = orc.accumulate_rho(g, p, q)
    if perturb:
        acc = acc * np.float32(1 + perturb)
    J = orc.unload_raw(g, acc)
    n3 = (g.nx, g.ny, g.nz)
    S = (g.nx + 2, g.ny + 2, g.nz + 2)
    Jg = J[:, :3].reshape(S[2], S[1], S[0], 3).transpose(2, 1, 0, 3).copy()  # [x,y,z,c]
    R = (rho1 - rho0).reshape(S[2], S[1], S[0]).transpose(2, 1, 0)
    per = [g.pbc[a] == 0 for a in range(3)]
    for a in range(3):  # fold periodic planes n+1 -> 1
        if per[a]:
            sl_hi = [slice(None)] * 3; sl_hi[a] = n3[a] + 1
            sl_lo = [slice(None)] * 3; sl_lo[a] = 1
            Jg[tuple(sl_lo)] += Jg[tuple(sl_hi)]
            Jg[tuple(sl_hi)] = 0
            R[tuple(sl_lo)] += R[tuple(sl_hi)]
            R[tuple(sl_hi)] = 0
    res = 4 * R
    for a in range(3):
        Ja = Jg[..., a]
        if per[a]:
            # J(n) - J(n - e) with periodic wrap over interior planes 1..n
            core = np.take(Ja, np.arange(1, n3[a] + 1), axis=a)
            div = core - np.roll(core, 1, axis=a)
            pad = np.zeros_like(Ja)
            put = [slice(None)] * 3; put[a] = slice(1, n3[a] + 1)
            pad[tuple(put)] = div
            res = res + pad
        else:
            shifted = np.zeros_like(Ja)
            s_dst = [slice(None)] * 3; s_dst[a] = slice(1, None)
            s_src = [slice(None)] * 3; s_src[a] = slice(0, -1)
            shifted[tuple(s_dst)] = Ja[tuple(s_src)]
            res = res + (Ja - shifted)
    return np.abs(res).max(), np.abs(4 * R).max(), p, acc


@pytest.mark.parametrize("seed", [0, 1])
def test_continuity_periodic(orc, seed):
    g = grid(n=4, dt=0.5)
    resid, scale, _, _ = _continuity(orc, g, 2000, seed, 0.05)
    assert scale > 1.0
    assert resid < 2e-5 * max(1.0, scale), (resid, scale)


def test_continuity_reflect_z(orc):
    g = grid(n=4, dt=0.5, pbc=(0, 0, 1, 0, 0, 1))
    resid, scale, p, _ = _continuity(orc, g, 2000, 7, 0.05)
    assert scale > 1.0
    assert resid < 2e-5 * max(1.0, scale)


def test_continuity_detects_wrong_current(orc):
    """Sanity of the pin itself: a 1% current error is caught."""
    g = grid(n=4, dt=0.5)
    resid, scale, _, _ = _continuity(orc, g, 2000, 3, 0.0, perturb=0.01)
    assert resid > 1e-3 * scale


def test_deposit_totals(orc):
    g = grid(n=5, dt=0.5)
    q = -0.7
    p = inputs.random_particles(g, 3000, 11, u_scale=0.9)
    interp = np.zeros((g.nv, 20), np.float32)
    acc = np.zeros((g.nv, 12), np.float32)
    acc_abs = np.zeros((g.nv, 12), np.float64)
    u = np.stack([p["ux"], p["uy"], p["uz"]], 1).astype(np.float64)
    gam = np.sqrt(1 + (u**2).sum(1))
    disp = u * 0.5 / gam[:, None]          # half displacement, cdt_dx = 0.5
    qw = q * p["w"].astype(np.float64)
    orc.advance_p(g, q, 1.0, p, interp, acc, acc_abs)
    for a in range(3):
        tot = acc[:, 4 * a:4 * a + 4].astype(np.float64).sum()
        exp = 4 * (qw * disp[:, a]).sum()
        assert abs(tot - exp) < 1e-5 * acc_abs[:, 4 * a:4 * a + 4].sum()


# ----------------------------------- TV2 / TV3 golden constants (c.5) --
def _golden():
    import json
    import os
    with open(os.path.join(os.path.dirname(__file__), "golden", "boris_tv2_tv3.json")) as fh:
        return json.load(fh)


def test_tv2_one_step_float32(orc):
    """TV2: one float32 step of the tan-corrected Boris equals the survey's
    float32 value (printed to 8 digits: 1 float32 ulp of slack)."""
    tv = _golden()["TV2_gyration"]
    g = grid(dt=tv["setup"]["dt"])
    p = one_particle(g, u=tuple(tv["setup"]["u0"]))
    us, _ = run(orc, g, p, uniform_fields(g, B=tuple(tv["setup"]["cB"])), 1.0, 1.0, 1, track=True)
    want = np.array(tv["u_after_one_step_float32"], np.float64)
    assert np.all(np.abs(us[0] - want) <= np.spacing(np.float32(0.3)).astype(np.float64) * 1.01), (us[0], want)


def test_tv2_discrete_rotation_angle_and_radius(orc):
    """TV2: the discrete rotation per step is theta = 2 atan(v3 |cB|) =
    0.7241304419859643 (not the continuous 2 phi = 0.72421; a dropped or
    extra tan-series term moves it by > 1e-5), and the orbit is the regular
    polygon of circumradius R = 0.3145545360723451 (not r_L = 0.30769)."""
    tv = _golden()["TV2_gyration"]
    g = grid(dt=tv["setup"]["dt"])
    p = one_particle(g, u=tuple(tv["setup"]["u0"]))
    us, xs = run(orc, g, p, uniform_fields(g, B=tuple(tv["setup"]["cB"])), 1.0, 1.0, 1000, track=True)
    ang = np.unwrap(np.arctan2(us[:, 1], us[:, 0]))
    theta = -(ang[-1] - ang[0]) / (len(ang) - 1)
    assert abs(theta - tv["theta_per_step"]) < 2e-7, theta
    assert abs(tv["two_phi"] - tv["theta_per_step"]) > 50 * 2e-7   # the pin discriminates
    a, b, c = xs[:-2, :2], xs[1:-1, :2], xs[2:, :2]
    la = np.linalg.norm(b - c, axis=1); lb = np.linalg.norm(a - c, axis=1); lc = np.linalg.norm(a - b, axis=1)
    area = 0.5 * np.abs((b - a)[:, 0] * (c - a)[:, 1] - (b - a)[:, 1] * (c - a)[:, 0])
    R = np.median(la * lb * lc / (4 * area))
    assert abs(R - tv["orbit_radius"]) / tv["orbit_radius"] < 1e-4, R
    assert abs(tv["larmor_radius_continuous"] - tv["orbit_radius"]) / tv["orbit_radius"] > 1e-2
    assert np.abs(np.linalg.norm(np.diff(xs, axis=0), axis=1) - tv["step_length"]).max() < 2e-6


def test_tv3_ExB_discrete_fixed_point(orc):
    """TV3: with E = (0, 0.01, 0), cB = (0, 0, 1), qdt_2mc = 0.3, the
    momentum u* = (0.009699099484663786, 0, 0) is a fixed point of the push
    (to float32 round-off over 1000 steps), while the textbook drift
    gamma E / cB = 0.0100005 is not (it gyrates about u*)."""
    tv = _golden()["TV3_ExB_fixed_point"]
    st = tv["setup"]
    g = grid(dt=st["dt"])
    fields = uniform_fields(g, E=tuple(st["E"]), B=tuple(st["cB"]))
    p = one_particle(g, u=(tv["ux_star"], 0.0, 0.0))
    us, _ = run(orc, g, p, fields, 1.0, 1.0, 1000, track=True)
    u0 = np.array([np.float32(tv["ux_star"]), 0.0, 0.0])
    assert np.abs(us - u0).max() < 2e-8, np.abs(us - u0).max()
    p = one_particle(g, u=(tv["textbook_gamma_E_over_B"], 0.0, 0.0))
    us2, _ = run(orc, g, p, fields, 1.0, 1.0, 20, track=True)
    assert np.abs(us2 - np.array([tv["textbook_gamma_E_over_B"], 0, 0])).max() > 1e-4


# ------------------------------------------- orc_remove_absorbed (R12) --
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_remove_absorbed_survivors(orc, seed):
    """Absorbing faces (reading R12): after a push, the particles stopped on
    an ABSORB face (p.i = 8 voxel + face, pbc[face] == absorb) are removed.
    Pinned without the oracle's back-fill: the survivors are exactly the
    multiset of particles NOT listed as absorbed movers, their count is np
    minus the absorbed ones, particles before the new end that were not
    removed keep their slot, and movers on a non-absorbing (remote) face
    are kept."""
    # absorb on -z/+z, remote (another rank) on +y: both produce movers
    g = inputs.GridSpec(6, 5, 4, dt=0.5, pbc=(0, 0, 2, 0, 0, 2), nbr_rank=(0, 0, 0, 0, 1, 0))
    p = inputs.random_particles(g, 4000, 40 + seed, u_scale=1.5)
    interp = orc.load_interpolator(g, np.zeros((g.nv, 8), np.float32))
    acc = np.zeros((g.nv, 12), np.float32)
    mv = orc.advance_p(g, -1.0, 1.0, p, interp, acc)
    face = p["i"][mv["idx"]] & 7
    absorbed = np.zeros(p.size, bool)
    absorbed[mv["idx"][(face == 2) | (face == 5)]] = True
    remote = mv["idx"][face == 4]
    assert absorbed.sum() > 50 and remote.size > 50
    before = p.copy()
    left = orc.remove_absorbed(g, p, mv)    # the survivors, back-filled in place
    assert len(left) == before.size - absorbed.sum()
    key = lambda a: np.sort(np.ascontiguousarray(a).view(np.dtype((np.void, 32))))
    assert np.array_equal(key(left), key(before[~absorbed]))
    keep = np.nonzero(~absorbed[:len(left)])[0]
    assert np.array_equal(left[keep].view(np.uint32), before[keep].view(np.uint32))
    # remote movers are still there (they leave through migration, not here)
    assert set(key(before[remote]).tolist()) <= set(key(left).tolist())


def test_move_deposit_replays_advance(orc):
    """orc_move_deposit (the replay tool of the FAST-mode parity tests) given
    the oracle's own pushed momenta reproduces orc_advance_p exactly."""
    g = inputs.GridSpec(6, 5, 4, dt=0.5, pbc=(0, 0, 2, 0, 0, 1))
    p = inputs.random_particles(g, 3000, 17, u_scale=1.2)
    interp = orc.load_interpolator(g, (np.random.default_rng(2).random((g.nv, 8), np.float32) - 0.5) * 0.2)
    acc = np.zeros((g.nv, 12), np.float32)
    p1 = p.copy()
    mv = orc.advance_p(g, -1.0, 1.0, p1, interp, acc)
    from parity_util import replay_inputs
    pr = replay_inputs(orc, g, -1.0, p, p1)     # the pushed momenta (reflections undone)
    assert (pr["uz"] != p1["uz"]).sum() > 0      # some particles were reflected
    acc_r = np.zeros_like(acc)
    mv_r = orc.move_deposit(g, -1.0, pr, acc_r)
    assert np.array_equal(pr.view(np.uint32), p1.view(np.uint32))
    assert np.array_equal(acc_r.view(np.uint32), acc.view(np.uint32))
    assert np.array_equal(mv_r.view(np.uint32), mv.view(np.uint32)) and mv.size > 0


@pytest.mark.parametrize("threads", [1, 3, 8])
def test_advance_p_omp_matches_serial(orc, threads):
    """The all-core baseline (orc_advance_p_omp: particle blocks, private
    accumulators) computes the serial oracle's step: particles bit-exact,
    accumulator equal up to summation order, same movers."""
    g = inputs.GridSpec(6, 5, 4, dt=0.5, pbc=(0, 0, 2, 0, 0, 2))
    p = inputs.random_particles(g, 5001, 23, u_scale=1.0)
    interp = orc.load_interpolator(g, (np.random.default_rng(4).random((g.nv, 8), np.float32) - 0.5) * 0.2)
    a1 = np.zeros((g.nv, 12), np.float32)
    aa = np.zeros((g.nv, 12), np.float64)
    p1 = p.copy()
    m1 = orc.advance_p(g, -1.0, 1.0, p1, interp, a1, aa)
    a2 = np.zeros_like(a1)
    p2 = p.copy()
    m2 = orc.advance_p_omp(g, -1.0, 1.0, p2, interp, a2, threads)
    assert np.array_equal(p1.view(np.uint32), p2.view(np.uint32))
    assert np.all(np.abs(a1.astype(np.float64) - a2) <= 1e-5 * aa + 1e-30)
    assert np.array_equal(np.sort(m1.view(np.uint32).reshape(-1, 4), axis=0),
                          np.sort(m2.view(np.uint32).reshape(-1, 4), axis=0)) and m1.size > 0


# ------------------------------------------------ gather / geometry pins --
def _edge_field_push(orc, comp, coef, g, p):
    """One step from rest with E only (B = 0): u = 2 qdt_2mc E(particle)."""
    f = np.zeros((g.nv, 8), np.float32)
    z, y, x = np.meshgrid(np.arange(g.nz + 2), np.arange(g.ny + 2), np.arange(g.nx + 2), indexing="ij")
    X = {"x": x, "y": y, "z": z}
    a, b, c, d, t1, t2 = coef
    f[:, comp] = (a + b * X[t1] + c * X[t2] + d * X[t1] * X[t2]).reshape(-1).astype(np.float32)
    interp = orc.load_interpolator(g, f)
    acc = np.zeros((g.nv, 12), np.float32)
    q = p.copy()
    orc.advance_p(g, 1.0, 1.0, q, interp, acc)
    return q


@pytest.mark.parametrize("comp,t1,t2", [(0, "y", "z"), (1, "z", "x"), (2, "x", "y")])
def test_gather_bilinear_E_closed_form(orc, comp, t1, t2):
    """The gather ("gather phase"): E_a on the a-edges of a voxel,
    bilinear in the two transverse coordinates, is interpolated exactly at
    the particle -- E_a(particle) = f(x_t1 + (1+d_t1)/2, x_t2 + (1+d_t2)/2) for
    edge values f(X_t1, X_t2) = a + b X_t1 + c X_t2 + d X_t1 X_t2 (edge a of
    voxel (x,y,z) sits at node coordinates (x_t1, x_t2) transversely).  One
    step from rest with B = 0 gives u_a = 2 qdt_2mc E_a exactly (to float)."""
    # walls (the caller owns their ghost planes: the field stays bilinear up
    # to the last edge), particles away from them (no reflection in a step)
    g = inputs.GridSpec(6, 5, 7, dt=0.5, pbc=(1,) * 6)   # non-cubic counts: no axis symmetry
    inner = [g.voxel(x, y, z) for z in range(2, 7) for y in range(2, 5) for x in range(2, 6)]
    p = inputs.random_particles(g, 400, 11, vox=inner)
    p["ux"] = p["uy"] = p["uz"] = 0
    coef = (0.01, 0.003, -0.002, 0.0007, t1, t2)
    q = _edge_field_push(orc, comp, coef, g, p)
    xyz = dict(zip("xyz", g.coords(p["i"])))
    off = {"x": p["dx"].astype(np.float64), "y": p["dy"].astype(np.float64), "z": p["dz"].astype(np.float64)}
    X1 = xyz[t1] + (1 + off[t1]) / 2
    X2 = xyz[t2] + (1 + off[t2]) / 2
    E = coef[0] + coef[1] * X1 + coef[2] * X2 + coef[3] * X1 * X2
    qdt_2mc = 0.5 / 2
    names = ("ux", "uy", "uz")
    assert np.abs(q[names[comp]] - 2 * qdt_2mc * E).max() < 3e-8
    for k in range(3):
        if k != comp:
            assert np.all(q[names[k]] == 0)


@pytest.mark.parametrize("axis", [0, 1, 2])
def test_gather_linear_B_closed_form(orc, axis):
    """cB_a is linear along its face normal inside the voxel: at the particle
    cB_a = cb(x_a + (1+d_a)/2) for face values cb(X_a) = a + b X_a.  A
    particle moving perpendicular to B rotates by theta = 2 atan(v3 |cB|)
    per step (pinned by TV2) -- checked against the closed-form |cB| at its
    position."""
    g = inputs.GridSpec(6, 5, 7, dt=0.5, pbc=(1,) * 6)
    inner = [g.voxel(x, y, z) for z in range(2, 7) for y in range(2, 5) for x in range(2, 6)]
    p = inputs.random_particles(g, 200, 12, vox=inner)
    names = ("ux", "uy", "uz")
    for k in range(3):
        p[names[k]] = 0
    perp = (axis + 1) % 3
    p[names[perp]] = 0.2
    f = np.zeros((g.nv, 8), np.float32)
    z, y, x = np.meshgrid(np.arange(g.nz + 2), np.arange(g.ny + 2), np.arange(g.nx + 2), indexing="ij")
    X = (x, y, z)[axis]
    f[:, 4 + axis] = (0.5 + 0.1 * X).reshape(-1).astype(np.float32)
    interp = orc.load_interpolator(g, f)
    acc = np.zeros((g.nv, 12), np.float32)
    q = p.copy()
    orc.advance_p(g, 1.0, 1.0, q, interp, acc)
    Xa = g.coords(p["i"])[axis] + (1 + p[("dx", "dy", "dz")[axis]].astype(np.float64)) / 2
    B = 0.5 + 0.1 * Xa
    qdt_2mc = 0.25
    gam = np.sqrt(1 + 0.04)
    v0 = qdt_2mc / gam
    v2 = v0 * v0 * B * B
    v3 = v0 * (1 + v2 * (1 / 3 + v2 * 2 / 15))
    theta = 2 * np.arctan(v3 * B)
    other = (axis + 2) % 3
    got = np.arctan2(np.abs(q[names[other]].astype(np.float64)), q[names[perp]].astype(np.float64))
    assert np.abs(got - theta).max() < 1e-5


def test_half_displacement_per_axis_on_noncubic_cells(orc):
    """The position advance uses c dt / d_a on each axis (VPIC's cdt_dx,
    cdt_dy, cdt_dz): on cells of 0.5 x 1 x 2 a particle at constant velocity
    moves u_a c dt / gamma physical units along each axis per step."""
    g = inputs.GridSpec(6, 5, 4, dx=0.5, dy=1.0, dz=2.0, dt=0.2)
    p = np.zeros(1, PD)
    p["i"] = g.voxel(3, 3, 2)
    p["ux"], p["uy"], p["uz"] = 0.3, -0.2, 0.25
    p["w"] = 1
    x0 = np.array([(p["dx"][0] + 1) / 2 * 0.5, (p["dy"][0] + 1) / 2 * 1.0, (p["dz"][0] + 1) / 2 * 2.0])
    interp = orc.load_interpolator(g, np.zeros((g.nv, 8), np.float32))
    acc = np.zeros((g.nv, 12), np.float32)
    q = p.copy()
    orc.advance_p(g, 1.0, 1.0, q, interp, acc)
    assert q["i"][0] == p["i"][0]
    x1 = np.array([(q["dx"][0] + 1) / 2 * 0.5, (q["dy"][0] + 1) / 2 * 1.0, (q["dz"][0] + 1) / 2 * 2.0])
    u = np.array([0.3, -0.2, 0.25])
    assert np.abs((x1 - x0) - u * 0.2 / np.sqrt(1 + u @ u)).max() < 1e-7


def test_track_ending_exactly_on_a_face_stays(orc):
    """Reading R13: a track whose end lands exactly on a face (d + 2 disp ==
    1 in float) is not a crossing -- the end of track wins the tie with 2:
    the particle stays in its voxel with the offset exactly +1."""
    g = grid(n=4, dt=0.5)
    f32 = np.float32
    disp = (f32(1.0) * f32(0.5)) * (f32(1.0) / np.sqrt(f32(1.0) + f32(1.0) * f32(1.0)))
    d = f32(1.0) - f32(2.0) * disp
    for _ in range(8):
        e = (d + disp) + disp
        if e == f32(1.0):
            break
        d = np.nextafter(d, f32(2.0) if e < 1 else f32(-2.0), dtype=np.float32)
    p = one_particle(g, d=(float(d), 0.0, 0.0), u=(1.0, 0.0, 0.0))
    interp = orc.load_interpolator(g, uniform_fields(g))
    acc = np.zeros((g.nv, 12), np.float32)
    v0 = p["i"][0]
    orc.advance_p(g, 1.0, 1.0, p, interp, acc)
    assert p["i"][0] == v0 and p["dx"][0] == np.float32(1.0)


def test_move_p_end_of_track_ties_with_two(orc):
    """Reading R13 inside move_p: a streak whose end lies exactly on a face
    (fraction to the face == 2, the end-of-track value) ends the move -- the
    particle stays in its voxel on the face, it does not cross (d = 0.5,
    remaining half-displacement 0.25: (1 - 0.5) / 0.25 = 2 exactly)."""
    g = grid(n=4, dt=0.5)
    acc = np.zeros((g.nv, 12), np.float32)
    for axis in range(3):
        d = [0.0, 0.0, 0.0]
        r = [0.0, 0.0, 0.0]
        d[axis], r[axis] = 0.5, 0.25
        p = one_particle(g, d=tuple(d))
        v0 = p["i"][0]
        mv = _mover(tuple(r))
        assert orc.move_p(g, p, mv, acc, 1.0) == 0
        assert p["i"][0] == v0
        assert (p["dx"][0], p["dy"][0], p["dz"][0])[axis] == np.float32(1.0)

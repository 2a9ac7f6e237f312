"""Comparison helpers for the GPU-vs-oracle parity tests (tolerances of
BASELINE.json north_star / SURVEY.md §8(c) c.4, restated in DESIGN.md)."""
import numpy as np

from paper_conf_sc_tanlta25_b200 import inputs

ULP1 = float(np.spacing(np.float32(1.0)))   # 2^-23
OFFSET_TOL = 4 * ULP1                       # 4 ulp(1.0) on the cell offsets


def global_pos(g, p):
    x, y, z = g.coords(p["i"].astype(np.int64))
    return np.stack([x + (1 + p["dx"].astype(np.float64)) / 2,
                     y + (1 + p["dy"].astype(np.float64)) / 2,
                     z + (1 + p["dz"].astype(np.float64)) / 2], -1)


def assert_particles_bitexact(a, b):
    va = np.ascontiguousarray(a).view(np.uint32).reshape(-1, 8)
    vb = np.ascontiguousarray(b).view(np.uint32).reshape(-1, 8)
    bad = np.nonzero((va != vb).any(1))[0]
    assert bad.size == 0, f"{bad.size} particles differ, first {bad[:5]}: {a[bad[:3]]} vs {b[bad[:3]]}"


def kick_bound(g, p, q, m, interp):
    """Upper bound of |2 qdt_2mc E| at each particle (|offsets| <= 1), from the
    interpolator coefficients of its voxel: the size of the E-kick terms that
    are added to and cancelled against u inside the push."""
    qdt_2mc = abs(q * g.dt / (2 * m * g.cvac))
    f = np.abs(interp[p["i"]].astype(np.float64))
    return 2 * qdt_2mc * np.stack([f[:, 0:4].sum(1), f[:, 4:8].sum(1), f[:, 8:12].sum(1)], 1)


def assert_particles_close(g, gpu, orc, u_old, kick=None):
    """Per particle, in the oracle's voxel frame (a face tie may put the GPU
    particle in the neighbouring voxel: compare global positions, periodic
    wrap folded): |d offset| <= 4 ulp(1); |du| <= max(4 ulp(u), 1e-6 max(|u|,
    |u_old|, |2 qdt_2mc E|)) -- the last term is the size of the intermediate
    sums when the E kick cancels u (tolerance reading T2)."""
    assert gpu.shape == orc.shape
    n = np.array([g.nx, g.ny, g.nz], np.float64)
    d = global_pos(g, gpu) - global_pos(g, orc)
    d = d - n * np.round(d / n)
    off_err = 2 * np.abs(d)   # offset units: 2 per cell
    assert off_err.max(initial=0) <= OFFSET_TOL, f"max offset err {off_err.max()}"
    need_kick = np.zeros(gpu.shape[0], bool)
    for k, c in enumerate(("ux", "uy", "uz")):
        ug, uo = gpu[c].astype(np.float64), orc[c].astype(np.float64)
        scale = np.maximum(np.abs(uo), np.abs(u_old[:, k]))
        base = np.maximum(4 * np.spacing(np.abs(orc[c])).astype(np.float64), 1e-6 * scale)
        if kick is not None:
            scale = np.maximum(scale, kick[:, k])
        tol = np.maximum(4 * np.spacing(np.abs(orc[c])).astype(np.float64), 1e-6 * scale)
        err = np.abs(ug - uo)
        need_kick |= err > base
        bad = np.nonzero(err > tol)[0]
        assert bad.size == 0, f"{c}: {bad.size} out of tol, worst {err[bad].max()} vs {tol[bad].min()}"
    assert np.array_equal(gpu["w"], orc["w"])
    return int(need_kick.sum())   # particles within T2 only thanks to its kick term


def assert_acc_close(acc_gpu, acc_orc, acc_abs, rel=1e-5, cond=None):
    """T1: |a_gpu - a_orc| <= rel * sum|contributions| per entry (atomic
    reordering only: the partials are equal because the streaks are).
    T3 (FAST mode, cond = the oracle's sum of |q uX| per entry): + rel * cond,
    the bound of T2's particle tolerance propagated through ACCUMULATE_J
    (T3).  Returns the number of entries that needed the T3 term."""
    err = np.abs(acc_gpu.astype(np.float64) - acc_orc.astype(np.float64))
    t1 = rel * acc_abs + 1e-30
    tol = t1 if cond is None else t1 + rel * cond
    bad = np.argwhere(err > tol)
    assert bad.size == 0, f"{len(bad)} acc entries out of tol; worst err {err.max()}, at {bad[:3]}"
    return int((err > t1).sum())


def u_of(p):
    return np.stack([p["ux"], p["uy"], p["uz"]], 1).astype(np.float64)


def replay_inputs(orc, g, q, p, p_gpu):
    """The particles with the GPU's PUSHED momenta (before the move): its
    final momenta, with the components a reflecting wall negated during the
    move negated back -- for each particle the one sign pattern (over the
    reflecting axes) whose oracle move ends in the GPU's final momentum and
    position."""
    refl = [a for a in range(3) if g.pbc[a] == inputs.BC_REFLECT or g.pbc[a + 3] == inputs.BC_REFLECT]
    comps = ("ux", "uy", "uz")
    chosen = np.full(p.size, -1)
    pr = p.copy()
    for c in comps:
        pr[c] = p_gpu[c]
    for pat in range(1 << len(refl)):
        cand = pr.copy()
        for b, a in enumerate(refl):
            if pat >> b & 1:
                cand[comps[a]] = -cand[comps[a]]
        out = cand.copy()
        orc.move_deposit(g, q, out, None)          # trajectories only
        ok = (out.view(np.uint32).reshape(-1, 8) == p_gpu.view(np.uint32).reshape(-1, 8)).all(1)
        pick = ok & (chosen < 0)
        chosen[pick] = pat
        if pat:
            for c in comps:
                pr[c][pick] = cand[c][pick]
    assert (chosen >= 0).all(), f"{(chosen < 0).sum()} GPU particles are no oracle move of any pushed momentum"
    return pr

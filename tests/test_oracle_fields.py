"""Pins for the oracle's field solver (VPIC advance_b /
advance_e; reading F1 in DESIGN.md).

* vacuum standing wave: with the VPIC split step advance_b(1/2),
  advance_e, advance_b(1/2) and B = 0 initially, every E mode evolves as
  E_n = cos(n w dt) E_0 with the discrete Yee/leapfrog dispersion
  cos(w dt) = 1 - 2 (c dt/d)^2 sin^2(k d / 2) -- for all six (propagation
  axis, E component) pairs, on non-cubic cells;
* advance_b keeps div B at round-off for any E (div curl = 0 on the Yee
  grid): any wrong index or sign in the curl breaks it;
* Gauss's law with a charge-conserving current: E advanced from E = B = 0 by
  the jf of one particle push changes div E by exactly the change of the
  cloud-in-cell charge density / eps0.
"""
import math

import numpy as np
import pytest

from paper_conf_sc_tanlta25_b200 import inputs



def step(orc, g, f, jf=None, eps0=1.0):
    orc.advance_b(g, f, 0.5)
    orc.advance_e(g, f, np.zeros((g.nv, 4), np.float32) if jf is None else jf, eps0)
    orc.advance_b(g, f, 0.5)


def as_grid(g, f):
    return f.reshape(g.nz + 2, g.ny + 2, g.nx + 2, 8)


@pytest.mark.parametrize("a", [0, 1, 2])
@pytest.mark.parametrize("b_off", [1, 2])
def test_standing_wave_dispersion(orc, a, b_off):
    b = (a + b_off) % 3          # E component, transverse to the wave vector axis a
    n = [4, 4, 4]
    n[a] = 24
    d = [0.7, 1.0, 1.3]
    dt = 0.9 / math.sqrt(sum(1 / x**2 for x in d))
    g = inputs.GridSpec(*n, dx=d[0], dy=d[1], dz=d[2], dt=dt)
    f = np.zeros((g.nv, 8), np.float32)
    F = as_grid(g, f)
    mode = 3
    k = 2 * math.pi * mode / (n[a] * d[a])
    idx = np.arange(n[a] + 2)                          # node index along a (E_b sits on nodes in a)
    prof = np.sin(k * (idx - 1) * d[a]).astype(np.float32)
    shape = [1, 1, 1]
    shape[2 - a] = n[a] + 2                             # array axes are (z, y, x)
    F[..., b] = prof.reshape(shape)
    E0 = F[1:-1, 1:-1, 1:-1, b].astype(np.float64).copy()
    lam = g.cvac * dt / d[a]
    cwdt = 1 - 2 * lam**2 * math.sin(k * d[a] / 2) ** 2
    wdt = math.acos(cwdt)
    for nstep in range(1, 61):
        step(orc, g, f)
        got = as_grid(g, f)[1:-1, 1:-1, 1:-1, b].astype(np.float64)
        exp = math.cos(nstep * wdt) * E0
        assert np.abs(got - exp).max() < 2e-5, (nstep, np.abs(got - exp).max())
        others = [c for c in range(3) if c != b]
        assert np.abs(as_grid(g, f)[1:-1, 1:-1, 1:-1][..., others]).max() < 1e-6
    # the mode really oscillated over the checked steps (a wrong sign would grow)
    assert min(math.cos(n * wdt) for n in range(1, 61)) < -0.5


def div_b(g, f):
    F = as_grid(g, f).astype(np.float64)
    c = F[1:-1, 1:-1, 1:-1]
    return ((F[1:-1, 1:-1, 2:, 4] - c[..., 4]) / g.dx + (F[1:-1, 2:, 1:-1, 5] - c[..., 5]) / g.dy
            + (F[2:, 1:-1, 1:-1, 6] - c[..., 6]) / g.dz)


def test_advance_b_keeps_div_b(orc):
    g = inputs.GridSpec(6, 5, 7, dx=0.8, dy=1.1, dz=0.9, dt=0.4)
    rng = np.random.default_rng(3)
    f = np.zeros((g.nv, 8), np.float32)
    scale = 0.0
    for it in range(20):
        f[:, 0:3] = rng.standard_normal((g.nv, 3)).astype(np.float32)  # fresh random E each time
        orc.advance_b(g, f, 0.5)
        # +ghost planes of cB must mirror plane 1 for the periodic divergence
        F = as_grid(g, f)
        F[:, :, g.nx + 1, 4:7] = F[:, :, 1, 4:7]
        F[:, g.ny + 1, :, 4:7] = F[:, 1, :, 4:7]
        F[g.nz + 1, :, :, 4:7] = F[1, :, :, 4:7]
        scale = max(scale, np.abs(F[..., 4:7]).max())
        assert np.abs(div_b(g, f)).max() < 1e-5 * scale / min(g.dx, g.dy, g.dz)
    assert scale > 1.0


def test_advance_b_detects_wrong_curl(orc):
    """Sanity of the pin: div of a non-curl field (random B) is not small."""
    g = inputs.GridSpec(6, 5, 7)
    f = np.zeros((g.nv, 8), np.float32)
    f[:, 4:7] = np.random.default_rng(1).standard_normal((g.nv, 3))
    assert np.abs(div_b(g, f)).max() > 0.1


def test_gauss_law_with_deposit(orc):
    d = (0.5, 1.0, 2.0)
    g = inputs.GridSpec(5, 4, 3, dx=d[0], dy=d[1], dz=d[2], dt=0.25)
    eps0, q = 1.7, -0.9
    p = inputs.random_particles(g, 3000, 12, u_scale=0.6)
    rho0 = orc.accumulate_rho(g, p, q)
    acc = np.zeros((g.nv, 12), np.float32)
    orc.advance_p(g, q, 1.0, p, np.zeros((g.nv, 20), np.float32), acc)
    rho1 = orc.accumulate_rho(g, p, q)
    jf = orc.unload_accumulator(g, acc)
    f = np.zeros((g.nv, 8), np.float32)
    orc.advance_e(g, f, jf, eps0)
    F = as_grid(g, f).astype(np.float64)
    # periodic backward divergence at nodes 1..n
    E = F[1:-1, 1:-1, 1:-1, :3]
    div = ((E[..., 0] - np.roll(E[..., 0], 1, axis=2)) / d[0] + (E[..., 1] - np.roll(E[..., 1], 1, axis=1)) / d[1]
           + (E[..., 2] - np.roll(E[..., 2], 1, axis=0)) / d[2])
    S = (g.nz + 2, g.ny + 2, g.nx + 2)
    drho = (rho1 - rho0).reshape(S)[1:-1, 1:-1, 1:-1] / (d[0] * d[1] * d[2])
    scale = np.abs(drho).max() / eps0
    assert scale > 0.1
    assert np.abs(div - drho / eps0).max() < 1e-4 * scale

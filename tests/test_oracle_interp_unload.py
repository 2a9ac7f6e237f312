"""Pins for load_interpolator and unload_accumulator (VPIC reading).

* Fields bilinear in the two coordinates transverse to an E component (and
  linear along the normal of a cB component) have closed-form interpolator
  coefficients: value at the cell centre and half-cell derivatives (the
  particle offset d in [-1,1] spans one cell, so d/dd = 1/2 d/dX).
* Uniform fields are reproduced bit-exactly.
* The periodic ghost fill copies plane 1 into plane n+1.
* unload: a single accumulator slot lands on exactly one Yee edge, with the
  factor c_axis = 1/(4 dA dt); a particle moving along x through the cell
  centre loads the 4 x-edges equally.
"""
import numpy as np
import pytest

from paper_conf_sc_tanlta25_b200 import inputs


def yee_fields(g, coef, rng=None):
    """ex(Y,Z) = a+bY+cZ+dYZ at x-edge (x+1/2, y, z) etc.; cbx(X) = a+bX at
    x-face (x, y+1/2, z+1/2) etc.  coef: dict of 4-tuples / 2-tuples."""
    v = np.arange(g.nv)
    x, y, z = [c.astype(np.float64) for c in g.coords(v)]
    f = np.zeros((g.nv, 8), np.float64)
    a, b, c, d = coef["ex"]; f[:, 0] = a + b * y + c * z + d * y * z
    a, b, c, d = coef["ey"]; f[:, 1] = a + b * z + c * x + d * z * x
    a, b, c, d = coef["ez"]; f[:, 2] = a + b * x + c * y + d * x * y
    a, b = coef["cbx"]; f[:, 4] = a + b * x
    a, b = coef["cby"]; f[:, 5] = a + b * y
    a, b = coef["cbz"]; f[:, 6] = a + b * z
    return f.astype(np.float32)


def test_bilinear_closed_form(orc):
    g = inputs.GridSpec(5, 4, 3, pbc=(1,) * 6)  # non-periodic: no ghost overwrite
    coef = {"ex": (0.5, 0.25, -0.125, 0.0625), "ey": (-0.25, 0.125, 0.5, -0.03125),
            "ez": (0.75, -0.5, 0.25, 0.125), "cbx": (0.3, 0.2), "cby": (-0.1, 0.05), "cbz": (0.2, -0.4)}
    f = yee_fields(g, coef)
    interp = orc.load_interpolator(g, f.copy()).astype(np.float64)
    vox = g.interior_voxels()
    x, y, z = [c.astype(np.float64) for c in g.coords(vox)]
    I = interp[vox]
    xc, yc, zc = x + 0.5, y + 0.5, z + 0.5
    a, b, c, d = coef["ex"]
    exp = [a + b * yc + c * zc + d * yc * zc, 0.5 * (b + d * zc), 0.5 * (c + d * yc), 0.25 * d + 0 * x]
    a, b, c, d = coef["ey"]
    exp += [a + b * zc + c * xc + d * zc * xc, 0.5 * (b + d * xc), 0.5 * (c + d * zc), 0.25 * d + 0 * x]
    a, b, c, d = coef["ez"]
    exp += [a + b * xc + c * yc + d * xc * yc, 0.5 * (b + d * yc), 0.5 * (c + d * xc), 0.25 * d + 0 * x]
    a, b = coef["cbx"]; exp += [a + b * xc, 0.5 * b + 0 * x]
    a, b = coef["cby"]; exp += [a + b * yc, 0.5 * b + 0 * x]
    a, b = coef["cbz"]; exp += [a + b * zc, 0.5 * b + 0 * x]
    exp = np.stack(exp, 1)
    assert np.abs(I[:, :18] - exp).max() < 2e-6 * max(1.0, np.abs(exp).max())
    assert np.all(I[:, 18:] == 0)


def test_uniform_bit_exact(orc):
    g = inputs.GridSpec(4, 4, 4)
    f = np.zeros((g.nv, 8), np.float32)
    vals = np.array([0.1, -0.7, 3.3, 0, 1e-3, -2.5, 0.77, 0], np.float32)
    f[:] = vals
    I = orc.load_interpolator(g, f)[g.interior_voxels()]
    for k, c in zip((0, 4, 8, 12, 14, 16), (0, 1, 2, 4, 5, 6)):
        assert np.all(I[:, k] == vals[c])
    for k in (1, 2, 3, 5, 6, 7, 9, 10, 11, 13, 15, 17):
        assert np.all(I[:, k] == 0)


def test_periodic_ghost_fill(orc):
    g = inputs.GridSpec(3, 4, 5)
    rng = np.random.default_rng(1)
    f = rng.random((g.nv, 8)).astype(np.float32)
    f0 = f.copy()
    orc.load_interpolator(g, f)
    F = f.reshape(g.nz + 2, g.ny + 2, g.nx + 2, 8)
    assert np.array_equal(F[:, :, g.nx + 1], F[:, :, 1])
    assert np.array_equal(F[:, g.ny + 1, :], F[:, 1, :])
    assert np.array_equal(F[g.nz + 1], F[1])
    # interior untouched
    F0 = f0.reshape(F.shape)
    assert np.array_equal(F[1:g.nz + 1, 1:g.ny + 1, 1:g.nx + 1], F0[1:g.nz + 1, 1:g.ny + 1, 1:g.nx + 1])


# Quadrant -> edge offsets (Yee geometry): jx[0..3] = (-y-z), (+y-z), (-y+z),
# (+y+z) edges of the cell; jy cyclic over (z, x); jz over (x, y).
EDGE = {0: [(0, 0, 0), (0, 1, 0), (0, 0, 1), (0, 1, 1)],
        1: [(0, 0, 0), (0, 0, 1), (1, 0, 0), (1, 0, 1)],
        2: [(0, 0, 0), (1, 0, 0), (0, 1, 0), (1, 1, 0)]}


@pytest.mark.parametrize("slot", range(12))
def test_unload_single_slot(orc, slot):
    g = inputs.GridSpec(4, 5, 6, dx=0.5, dy=2.0, dz=1.5, dt=0.25, pbc=(1,) * 6)
    acc = np.zeros((g.nv, 12), np.float32)
    cell = (2, 3, 4)
    acc[g.voxel(*cell), slot] = 1.0
    jf = orc.unload_accumulator(g, acc)
    axis, quad = slot // 4, slot % 4
    off = EDGE[axis][quad]
    tgt = g.voxel(cell[0] + off[0], cell[1] + off[1], cell[2] + off[2])
    cfac = [0.25 / (g.dy * g.dz * g.dt), 0.25 / (g.dz * g.dx * g.dt), 0.25 / (g.dx * g.dy * g.dt)][axis]
    nz = np.argwhere(jf != 0)
    assert nz.tolist() == [[tgt, axis]]
    assert abs(jf[tgt, axis] - cfac) < 1e-6 * cfac


def test_particle_through_centre(orc):
    """A particle moving along +x through the cell centre: equal current on the
    4 x-edges, nothing on y/z edges."""
    g = inputs.GridSpec(4, 4, 4, dt=0.5, pbc=(1,) * 6)
    p = np.zeros(1, inputs.PARTICLE_DTYPE)
    p["i"] = g.voxel(2, 2, 2)
    p["dx"] = -0.5
    p["ux"] = 0.3
    p["w"] = 1.0
    acc = np.zeros((g.nv, 12), np.float32)
    orc.advance_p(g, 1.0, 1.0, p, np.zeros((g.nv, 20), np.float32), acc)
    a = acc[g.voxel(2, 2, 2)]
    assert np.all(a[0:4] == a[0]) and a[0] > 0
    assert np.all(a[4:] == 0)
    jf = orc.unload_accumulator(g, acc)
    nzx = sorted(np.nonzero(jf[:, 0])[0].tolist())
    assert nzx == sorted(g.voxel(2, 2 + dy, 2 + dz) for dy in (0, 1) for dz in (0, 1))
    assert np.all(jf[:, 1:] == 0)


def test_unload_periodic_fold(orc):
    g = inputs.GridSpec(3, 3, 3)
    rng = np.random.default_rng(2)
    acc = np.zeros((g.nv, 12), np.float32)
    acc[g.interior_voxels()] = rng.random((27, 12)).astype(np.float32)
    jf = orc.unload_accumulator(g, acc)
    gn = inputs.GridSpec(3, 3, 3, pbc=(1,) * 6)
    raw = orc.unload_accumulator(gn, acc).astype(np.float64)
    # total current conserved by the fold; ghost planes mirror plane 1
    J = jf.reshape(5, 5, 5, 4)
    R = raw.reshape(5, 5, 5, 4)
    assert abs(J[1:4, 1:4, 1:4, :3].sum() - R[1:5, 1:5, 1:5, :3].sum()) < 1e-4
    assert np.array_equal(J[:, :, 4], J[:, :, 1])
    assert np.array_equal(J[:, 4, :], J[:, 1, :])
    assert np.array_equal(J[4], J[1])

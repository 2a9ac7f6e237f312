"""Pins for orc_accumulate_rho (cloud-in-cell node charge, reading D1 in
DESIGN.md; VPIC accumulate_rho_p, ref. [3]) -- the reference the GPU
diagnostic vpic_accumulate_rho is checked against.

* corners: a particle at offsets (-1,-1,-1) puts all of q w on node (x,y,z),
  at (+1,+1,+1) on node (x+1,y+1,z+1) (node 1 when x = n on a periodic axis);
  at the cell centre q w / 8 on each of the 8 nodes;
* total charge: sum over nodes = q sum w (the CIC weights sum to 1);
* first moment (non-periodic axes): sum rho * node = q sum w * (x + (1 + dx)/2)
  per axis -- a swapped (1 - d) / (1 + d) or a wrong node index fails it.
"""
import numpy as np
import pytest

from paper_conf_sc_tanlta25_b200 import inputs


def one(g, x, y, z, d, w=1.0):
    p = np.zeros(1, inputs.PARTICLE_DTYPE)
    p["i"] = g.voxel(x, y, z)
    p["dx"], p["dy"], p["dz"] = d
    p["w"] = w
    return p


@pytest.mark.parametrize("pbc", [(0,) * 6, (1,) * 6], ids=["periodic", "reflect"])
def test_rho_corners_and_centre(orc, pbc):
    g = inputs.GridSpec(4, 3, 5, pbc=pbc)
    q = -0.75
    r = orc.accumulate_rho(g, one(g, 2, 1, 3, (-1, -1, -1), 2.0), q)
    assert r[g.voxel(2, 1, 3)] == q * 2.0 and np.count_nonzero(r) == 1
    r = orc.accumulate_rho(g, one(g, 4, 3, 5, (1, 1, 1), 2.0), q)
    node = g.voxel(1, 1, 1) if pbc[0] == 0 else g.voxel(5, 4, 6)
    assert r[node] == q * 2.0 and np.count_nonzero(r) == 1
    r = orc.accumulate_rho(g, one(g, 2, 2, 2, (0, 0, 0), 1.0), q)
    nodes = [g.voxel(2 + a, 2 + b, 2 + c) for a in (0, 1) for b in (0, 1) for c in (0, 1)]
    assert np.all(r[nodes] == q / 8) and np.count_nonzero(r) == 8


@pytest.mark.parametrize("pbc", [(0,) * 6, (1,) * 6, (0, 0, 1, 0, 0, 1)])
def test_rho_total_charge(orc, pbc):
    g = inputs.GridSpec(6, 5, 4, pbc=pbc)
    p = inputs.random_particles(g, 5000, 3)
    q = 1.3
    r = orc.accumulate_rho(g, p, q)
    tot = float(np.float32(q)) * p["w"].astype(np.float64).sum()   # the oracle takes q as float32
    assert abs(r.sum() - tot) < 1e-12 * abs(tot)


def test_rho_first_moment(orc):
    g = inputs.GridSpec(6, 5, 4, pbc=(1,) * 6)
    p = inputs.random_particles(g, 4000, 5)
    q = -0.4
    r = orc.accumulate_rho(g, p, q)
    S = (g.nx + 2, g.ny + 2, g.nz + 2)
    R = r.reshape(S[2], S[1], S[0]).transpose(2, 1, 0)
    xyz = np.stack(g.coords(p["i"].astype(np.int64)), 1).astype(np.float64)
    d = np.stack([p["dx"], p["dy"], p["dz"]], 1).astype(np.float64)
    w = p["w"].astype(np.float64)
    for a in range(3):
        pos = np.arange(S[a], dtype=np.float64)
        shape = [1, 1, 1]
        shape[a] = S[a]
        moment = (R * pos.reshape(shape)).sum()
        exp = float(np.float32(q)) * (w * (xyz[:, a] + (1 + d[:, a]) / 2)).sum()
        assert abs(moment - exp) < 1e-11 * abs(exp)


# ------------------------------------ orc_continuity_residual (reading D1) --
def _node_range(g):
    per = [g.pbc[a] == 0 and g.pbc[a + 3] == 0 for a in range(3)]
    return [range(1, (g.nx, g.ny, g.nz)[a] + (0 if per[a] else 1) + 1) for a in range(3)], per


@pytest.mark.parametrize("pbc", [(0,) * 6, (0, 0, 1, 0, 0, 1)], ids=["periodic", "reflect_z"])
def test_continuity_residual_definition(orc, pbc):
    """Hand cases: a charge change at one node gives d rho / (dV dt) there
    and nothing elsewhere; one jf edge value J on the x-edge of node n gives
    +J/dx at n and -J/dx at n + e_x (wrapped on a periodic axis)."""
    g = inputs.GridSpec(4, 3, 3, dx=0.5, dy=1.0, dz=2.0, dt=0.25, pbc=pbc)
    z = np.zeros(g.nv, np.float32)
    jf = np.zeros((g.nv, 4), np.float32)
    r1 = z.copy()
    r1[g.voxel(2, 2, 2)] = 3.0
    res, mag = orc.continuity_residual(g, z, r1, jf)
    (X, Y, Z), per = _node_range(g)
    inside = np.zeros(g.nv, bool)
    for zz in Z:
        for yy in Y:
            for xx in X:
                inside[g.voxel(xx, yy, zz)] = True
    assert np.all(np.isnan(res[~inside]))
    exp = np.zeros(g.nv)
    exp[g.voxel(2, 2, 2)] = 3.0 / (0.5 * 1.0 * 2.0 * 0.25)
    assert np.allclose(res[inside], exp[inside], rtol=0, atol=1e-12)
    # jf_x on the edge from node (4,1,1) (periodic: its +x node is (1,1,1))
    jf[g.voxel(4, 1, 1), 0] = 1.5
    res, _ = orc.continuity_residual(g, z, z, jf)
    assert res[g.voxel(4, 1, 1)] == pytest.approx(1.5 / 0.5)
    assert res[g.voxel(1, 1, 1)] == pytest.approx(-1.5 / 0.5)
    jf[:] = 0
    jf[g.voxel(2, 3, 1), 2] = -0.8           # z-edge from node (2,3,1) to (2,3,2)
    res, _ = orc.continuity_residual(g, z, z, jf)
    assert res[g.voxel(2, 3, 1)] == pytest.approx(-0.8 / 2.0)
    assert res[g.voxel(2, 3, 2)] == pytest.approx(0.8 / 2.0)
    assert np.nansum(np.abs(res)) == pytest.approx(0.8)


def test_continuity_residual_of_oracle_step(orc):
    """The oracle's own push: residual at float32 round-off of |drho/dt|;
    a 1% current error is detected (the pin discriminates)."""
    g = inputs.GridSpec(6, 5, 4, dt=0.4)
    p = inputs.random_particles(g, 20000, 3, u_scale=0.8)
    q = 0.7
    interp = orc.load_interpolator(g, np.zeros((g.nv, 8), np.float32))
    rho0 = orc.accumulate_rho(g, p, q).astype(np.float32)
    acc = np.zeros((g.nv, 12), np.float32)
    orc.advance_p(g, q, 1.0, p, interp, acc)
    rho1 = orc.accumulate_rho(g, p, q).astype(np.float32)
    jf = orc.unload_accumulator(g, acc)
    res, mag = orc.continuity_residual(g, rho0, rho1, jf)
    scale = np.nanmax(np.abs((rho1 - rho0).astype(np.float64))) / (g.dx * g.dy * g.dz * g.dt)
    assert np.nanmax(np.abs(res)) < 1e-4 * scale
    res2, _ = orc.continuity_residual(g, rho0, rho1, jf * np.float32(1.01))
    assert np.nanmax(np.abs(res2)) > 3e-3 * scale

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

"""Parity at full size for BASELINE.json configs[2] -- the Harris sheet,
256x128x128 cells, 2 species x 100 ppc mean (2 x 419,430,400 particles), a
sech^2 sheet of ~369 ppc over a ~62 ppc background, reflecting z walls: the
contention workload -- in the launch configuration bench.py times
(FAST math, AUTO deposit, TMA kernel).  One PIC step without the sort, so GPU
particle i is input particle i:

* particles: 2^16 sampled per species, recomputed one by one by the oracle;
* accumulators: voxels at the sheet centre, at both walls and at random,
  recomputed by the oracle from every particle that starts in the 3x3x3 block
  around the voxel (the only ones that can deposit into it).
"""
import numpy as np
import pytest
import torch

from paper_conf_sc_tanlta25_b200 import inputs
from parity_util import (assert_acc_close, assert_particles_bitexact, assert_particles_close, kick_bound,
                         replay_inputs, u_of)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def harris(orc):
    from paper_conf_sc_tanlta25_b200 import _build, vpic
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    _build.build()
    wl = inputs.config(2)
    g = wl.grid
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, wl.field_amp, kind="harris")
    hp = HotPath(wl, parts, fields, order=vpic.VPIC_SORT_STANDARD, math=vpic.MATH_FAST,
                 deposit=vpic.DEP_AUTO)
    hp.step(do_sort=False)
    torch.cuda.synchronize()
    interp_o = orc.load_interpolator(g, fields.copy())
    yield dict(wl=wl, g=g, parts=parts, hp=hp, interp_o=interp_o, vpic=vpic)
    hp.close()


def test_harris_fullsize_particles_sampled(orc, harris):
    wl, g, hp, interp_o = harris["wl"], harris["g"], harris["hp"], harris["interp_o"]
    rng = np.random.default_rng(3)
    for k, sp in enumerate(wl.species):
        p0 = harris["parts"][k]
        assert hp.species[k].np == p0.size          # reflecting walls: nobody leaves
        idx = np.sort(rng.choice(p0.size, 1 << 16, replace=False))
        got = harris["vpic"].particles_to_host(hp.species[k].p[torch.from_numpy(idx).cuda()])
        ps = p0[idx].copy()
        acc = np.zeros((g.nv, 12), np.float32)
        orc.advance_p(g, sp.q, sp.m, ps, interp_o, acc)
        assert_particles_close(g, got, ps, u_of(p0[idx]), kick_bound(g, p0[idx], sp.q, sp.m, interp_o))
        # T3: the move is the oracle's given the pushed momenta, bit for bit
        pr = replay_inputs(orc, g, sp.q, p0[idx].copy(), got)
        orc.move_deposit(g, sp.q, pr, None)
        assert_particles_bitexact(got, pr)


def test_harris_fullsize_accumulator_sampled(orc, harris):
    wl, g, hp, interp_o = harris["wl"], harris["g"], harris["hp"], harris["interp_o"]
    rng = np.random.default_rng(4)
    cells = [(1, 1, 64), (128, 64, 65), (200, 128, 1), (7, 99, 128)]
    cells += [tuple(int(c) for c in rng.integers(1, (g.nx + 1, g.ny + 1, g.nz + 1))) for _ in range(4)]
    for (x, y, z) in cells:
        block = [g.voxel((x - 1 + dx) % g.nx + 1, (y - 1 + dy) % g.ny + 1, z + dz)
                 for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)
                 if 1 <= z + dz <= g.nz]
        acc = np.zeros((g.nv, 12), np.float32)
        aabs = np.zeros((g.nv, 12), np.float64)
        for k, sp in enumerate(wl.species):
            p0 = harris["parts"][k]
            ps = p0[np.isin(p0["i"], np.array(block, np.int32))].copy()
            orc.advance_p(g, sp.q, sp.m, ps, interp_o, acc, aabs)
        v = g.voxel(x, y, z)
        got = hp.acc[v].cpu().numpy()[None]
        assert aabs[v].sum() > 0
        assert_acc_close(got, acc[v][None], aabs[v][None])

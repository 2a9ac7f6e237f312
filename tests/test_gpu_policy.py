"""The AUTO deposit policy inside a PIC run (pic.HotPath):
a sort period of a hot two-species plasma on a grid large enough for the
TMA kernel's pair/carry schedule and tensor-map stages, run with the policy
(WARP, then DEP_SMEM for the electrons from 0.4 cell of spread, WARP again
past 1.3) and with WARP throughout.  The deposit strategy only reorders the
current sums: particles bit-identical, jf within the atomic tolerance, and
the policy must really have switched."""
import numpy as np
import pytest
import torch

from paper_conf_sc_tanlta25_b200 import inputs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def V():
    from paper_conf_sc_tanlta25_b200 import _build, vpic
    _build.build()
    vpic.load()
    return vpic


def test_auto_policy_run_equals_warp_run(V):
    from paper_conf_sc_tanlta25_b200 import pic
    g = inputs.GridSpec(32, 24, 16)
    wl = inputs.Workload("policy", g, [inputs.Species("electron", -1.0, 1.0, 0.2, (0.3, 0.0, 0.0)),
                                       inputs.Species("ion", 1.0, 25.0, 0.02)], 64, 14, 14)
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, 0.02, kind="lpi")
    sched = [pic.auto_deposit_mode(0.2, g.cvac, g.dt, 1.0, k) for k in range(wl.steps)]
    assert V.DEP_SMEM in sched and sched[0] == V.DEP_WARP and sched[-1] == V.DEP_WARP
    runs = []
    for dep in (V.DEP_AUTO, V.DEP_WARP):
        hp = pic.HotPath(wl, parts, fields, deposit=dep, math=V.MATH_FAST)
        modes = []
        real = hp._set_deposit

        def spy(k, real=real, hp=hp, modes=modes):
            real(k)
            modes.append(hp._dep_mode)
        hp._set_deposit = spy
        hp.cycle(wl.steps)
        torch.cuda.synchronize()
        runs.append((hp, modes))
    (a, ma), (b, mb) = runs
    assert V.DEP_SMEM in ma and set(mb) == {V.DEP_WARP}
    for k in range(2):
        assert np.array_equal(a.particles_host(k).view(np.uint32), b.particles_host(k).view(np.uint32))
    vox = g.interior_voxels()
    ja, jb = a.jf.cpu().numpy()[vox], b.jf.cpu().numpy()[vox]
    assert np.abs(ja - jb).max() <= 1e-5 * np.abs(ja).max() * 8

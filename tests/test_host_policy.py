"""Host-side logic of pic.HotPath that runs without a GPU: the AUTO deposit
policy (DEP_SMEM while a species' thermal spread since its
sort is within [SMEM_SIGMA, SMEM_SIGMA_MAX) cells) and the NUMA binding
helper's no-GPU behaviour."""
from paper_conf_sc_tanlta25_b200 import inputs, pic, vpic


def schedule(sp, g, steps=20):
    return [pic.auto_deposit_mode(sp.u_th, g.cvac, g.dt, min(g.dx, g.dy, g.dz), k) for k in range(steps)]


def test_c2_electrons_switch_at_step_8_ions_never():
    wl = inputs.config(1)
    el, ion = wl.species
    s_el = schedule(el, wl.grid)
    # u_th 0.1, c dt / dx = 0.548: spread 0.0548 per step -> 0.4 cell at step 8
    assert s_el[:8] == [vpic.DEP_WARP] * 8 and s_el[8:] == [vpic.DEP_SMEM] * 12
    assert schedule(ion, wl.grid) == [vpic.DEP_WARP] * 20


def test_hot_lpi_electrons_return_to_warp():
    wl = inputs.config(4)
    el = wl.species[0]             # u_th 0.2: 0.4 cell at step 4, 1.3 cells at step 12
    s = schedule(el, wl.grid)
    assert s[:4] == [vpic.DEP_WARP] * 4
    assert s[4:12] == [vpic.DEP_SMEM] * 8
    assert s[12:] == [vpic.DEP_WARP] * 8


def test_bind_without_gpu_is_a_no_op():
    import os
    import torch
    before = os.sched_getaffinity(0)
    if not torch.cuda.is_available():
        assert pic.bind_to_gpu_cpus(0) is None
    assert os.sched_getaffinity(0) == before or torch.cuda.is_available()

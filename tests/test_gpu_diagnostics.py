"""GPU parity of the on-line charge-conservation diagnostics (SURVEY.md §8(f)
f4; reading D1): vpic_accumulate_rho against orc_accumulate_rho, and
vpic_continuity_residual on the GPU's own advance (the discrete continuity
invariant of the charge-conserving deposit, BASELINE north_star).

Tolerances: rho is a float32 sum of positive-weight contributions (per node
at most 8 x ppc of them), so |rho_gpu - rho_orc| <= 2e-5 * sum|contrib| (the
T1 form); the residual of float32 rho / jf is bounded by the cancellation in
rho1 - rho0, a few 1e-5 of max|drho/dt| -- checked at 3e-4, while a 1% current
error must show above 3e-3.
"""
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
    assert torch.cuda.is_available(), "gpu tests need a B200"
    return vpic


def rho_cases():
    out = []
    wl = inputs.config(0)
    pe = inputs.make_species_particles(wl)[0]
    out.append(("c1_sorted", wl.grid, pe))                       # warp-summed path
    out.append(("c1_shuffled", wl.grid, inputs.shuffle(pe, 3)))  # per-lane path
    g = inputs.GridSpec(7, 5, 4, dx=0.7, dz=1.2, pbc=(0, 0, 1, 0, 0, 1))
    out.append(("reflect_z_ragged", g, inputs.random_particles(g, 8193, 2)))
    g = inputs.GridSpec(5, 4, 3, pbc=(1,) * 6)
    out.append(("walls_one_voxel", g, inputs.random_particles(g, 4000, 4, vox=[g.voxel(5, 4, 3)])))
    out.append(("single", g, inputs.random_particles(g, 1, 5)))
    return out


@pytest.mark.parametrize("case", rho_cases(), ids=lambda c: c[0])
def test_rho_parity(V, orc, case):
    name, g, p = case
    q = -0.8
    ctx = V.Context(g)
    rho = torch.zeros(g.nv, dtype=torch.float32, device="cuda")
    V.vpic_accumulate_rho(ctx, q, V.particles_to_device(p), p.size, rho)
    got = rho.cpu().numpy().astype(np.float64)
    exp = orc.accumulate_rho(g, p, q)
    ab = orc.accumulate_rho(g, p, abs(q))      # weights are positive: sum |contrib|
    assert np.all(np.abs(got - exp) <= 2e-5 * ab + 1e-30), np.abs(got - exp).max()
    assert np.array_equal(got != 0, exp != 0)   # same support (folded nodes stay empty)


def test_rho_empty_and_invalid(V):
    g = inputs.GridSpec(4, 4, 4)
    ctx = V.Context(g)
    rho = torch.zeros(g.nv, dtype=torch.float32, device="cuda")
    p = V.particles_to_device(inputs.random_particles(g, 4, 1))
    V.vpic_accumulate_rho(ctx, 1.0, p, 0, rho)
    torch.cuda.synchronize()
    assert float(rho.abs().sum()) == 0.0
    with pytest.raises(V.VpicError):
        V.vpic_accumulate_rho(ctx, 1.0, p, -1, rho)
    with pytest.raises(V.VpicError):
        V.vpic_accumulate_rho(ctx, 1.0, None, 4, rho)


def advance_with_residual(V, g, p, q, fields, perturb=1.0, arrays=False):
    ctx = V.Context(g)
    ctx.set_option(V.VPIC_OPT_MATH, V.MATH_FAST)
    fd = torch.from_numpy(fields.copy()).cuda()
    interp = torch.zeros((g.nv, 24), dtype=torch.float32, device="cuda")
    V.vpic_load_interpolator(ctx, fd, interp)
    acc = torch.empty((g.nv, 12), dtype=torch.float32, device="cuda")
    V.vpic_clear_accumulator(ctx, acc)
    pd = V.particles_to_device(p)
    rho0 = torch.zeros(g.nv, dtype=torch.float32, device="cuda")
    rho1 = torch.zeros_like(rho0)
    V.vpic_accumulate_rho(ctx, q, pd, p.size, rho0)
    movers = torch.zeros((p.size, 4), dtype=torch.float32, device="cuda")
    nm = torch.zeros(1, dtype=torch.int64, device="cuda")
    V.vpic_advance_p(ctx, q, 1.0, pd, p.size, interp, acc, movers, p.size, nm, None)
    V.vpic_accumulate_rho(ctx, q, pd, p.size, rho1)
    jf = torch.empty((g.nv, 4), dtype=torch.float32, device="cuda")
    V.vpic_unload_accumulator(ctx, acc, jf)
    if perturb != 1.0:
        jf *= perturb
    out = torch.empty(2, dtype=torch.float32, device="cuda")
    res = torch.full((g.nv,), 7.0, dtype=torch.float32, device="cuda")
    V.vpic_continuity_residual(ctx, rho0, rho1, jf, out, res)
    torch.cuda.synchronize()
    if arrays:
        return (out.cpu().numpy().astype(np.float64), res.cpu().numpy(), rho0.cpu().numpy(),
                rho1.cpu().numpy(), jf.cpu().numpy())
    return out.cpu().numpy().astype(np.float64), res.cpu().numpy(), int(nm.item())


@pytest.mark.parametrize("pbc", [(0,) * 6, (0, 0, 1, 0, 0, 1)], ids=["periodic", "reflect_z"])
def test_continuity_residual_of_gpu_advance(V, pbc):
    g = inputs.GridSpec(8, 6, 5, dx=0.8, dy=1.0, dz=1.25, dt=0.4, pbc=pbc)
    p = inputs.random_particles(g, 60000, 21, u_scale=0.8)
    out, res, nm = advance_with_residual(V, g, p, 0.7, inputs.make_fields(g, 0.05))
    assert nm == 0
    rmax, scale = out
    assert scale > 1.0
    assert rmax < 3e-4 * scale, (rmax, scale)
    # the kernel's max agrees with the per-node residual it wrote
    ex = g.nx + (pbc[0] != 0)
    S = (g.nx + 2, g.ny + 2, g.nz + 2)
    R = res.reshape(S[2], S[1], S[0])
    core = R[1:g.nz + 1 + (pbc[2] != 0), 1:g.ny + 1 + (pbc[1] != 0), 1:ex + 1]
    assert np.abs(core).max() == np.float32(rmax)
    assert np.all(R[0] == 7.0)                    # nodes outside the range untouched


def test_continuity_residual_detects_wrong_current(V):
    g = inputs.GridSpec(8, 6, 5, dt=0.4)
    p = inputs.random_particles(g, 60000, 22, u_scale=0.8)
    out, _, _ = advance_with_residual(V, g, p, 0.7, inputs.make_fields(g, 0.05), perturb=1.01)
    assert out[0] > 3e-3 * out[1]



@pytest.mark.parametrize("pbc", [(0,) * 6, (0, 0, 1, 0, 0, 1)], ids=["periodic", "reflect_z"])
def test_continuity_residual_parity(V, orc, pbc):
    """vpic_continuity_residual against the oracle's definition
    (orc_continuity_residual, reading D1) on the same float32 rho0 / rho1 /
    jf: per node within 4 float32 roundings of the terms' magnitude, the
    same node range, the max reductions equal to the maxima of the arrays."""
    g = inputs.GridSpec(8, 6, 5, dx=0.8, dy=1.0, dz=1.25, dt=0.4, pbc=pbc)
    p = inputs.random_particles(g, 60000, 23, u_scale=0.8)
    out, res, rho0, rho1, jf = advance_with_residual(V, g, p, 0.7, inputs.make_fields(g, 0.05), arrays=True)
    ro, mag = orc.continuity_residual(g, rho0, rho1, jf)
    inside = ~np.isnan(ro)
    assert np.all(res[~inside] == 7.0)               # untouched outside the node range
    err = np.abs(res[inside].astype(np.float64) - ro[inside])
    assert np.all(err <= 4 * 2.0**-24 * mag[inside] + 1e-30), err.max()
    assert out[0] == np.float32(np.abs(res[inside]).max())
    drho = np.abs((rho1 - rho0).astype(np.float32) * np.float32(1.0 / (0.8 * 1.0 * 1.25 * 0.4)))
    assert abs(out[1] - drho[inside].max()) <= 4 * 2.0**-24 * drho[inside].max()

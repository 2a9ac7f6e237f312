"""Parity at BASELINE.json's full size, in the launch configuration bench.py
times (configs[1]: uniform 128^3, 128 ppc/species, 2 species = 2^29
particles; FAST math, AUTO deposit, standard order).

* particles: a random sample of 2^16 per species recomputed one by one by the
  oracle from the same inputs;
* accumulators: sampled voxels recomputed by the oracle from every particle
  that can deposit into them (the 3x3x3 block of cells around the voxel);
* sort (strided, tiled strided, standard) of the advanced electrons: the
  properties that define each order uniquely at any size -- a permutation,
  keys/counts consistent, and (k, input index) / (r, k) / (floor(k/T), r, k)
  strictly increasing.
"""
import numpy as np
import pytest
import torch

from paper_conf_sc_tanlta25_b200 import inputs
from parity_util import (assert_acc_close, assert_particles_bitexact, assert_particles_close, kick_bound,
                         replay_inputs, u_of)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def state(orc):
    from paper_conf_sc_tanlta25_b200 import _build, vpic
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    _build.build()
    wl = inputs.config(1)
    g = wl.grid
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, wl.field_amp, kind=wl.kind)
    hp = HotPath(wl, parts, fields, order=vpic.VPIC_SORT_STANDARD, math=vpic.MATH_FAST,
                 deposit=vpic.DEP_AUTO)
    hp.step(do_sort=True)      # sort (identity on the cell-major quiet start) + one PIC step
    torch.cuda.synchronize()
    interp_o = orc.load_interpolator(g, fields.copy())
    yield dict(wl=wl, g=g, parts=parts, fields=fields, hp=hp, interp_o=interp_o, vpic=vpic)
    hp.close()


def test_fullsize_particles_sampled(orc, state):
    wl, g, hp, interp_o = state["wl"], state["g"], state["hp"], state["interp_o"]
    rng = np.random.default_rng(1)
    for k, sp in enumerate(wl.species):
        p0 = state["parts"][k]
        idx = np.sort(rng.choice(p0.size, 1 << 16, replace=False))
        got = state["vpic"].particles_to_host(hp.species[k].p[torch.from_numpy(idx).cuda()])
        ps = p0[idx].copy()
        acc = np.zeros((g.nv, 12), np.float32)
        orc.advance_p(g, sp.q, sp.m, ps, interp_o, acc)
        assert_particles_close(g, got, ps, u_of(p0[idx]), kick_bound(g, p0[idx], sp.q, sp.m, interp_o))
        # T3: the bench arithmetic's move is the oracle's given the pushed
        # momenta -- every sampled particle's position and voxel bit for bit
        pr = replay_inputs(orc, g, sp.q, p0[idx].copy(), got)
        orc.move_deposit(g, sp.q, pr, None)
        assert_particles_bitexact(got, pr)


def test_fullsize_accumulator_sampled(orc, state):
    wl, g, hp, interp_o = state["wl"], state["g"], state["hp"], state["interp_o"]
    acc_gpu = hp.acc
    rng = np.random.default_rng(2)
    cells = [(1, 1, 1), (128, 128, 128), (64, 1, 128)] + [tuple(rng.integers(1, 129, 3)) for _ in range(5)]
    ppc = wl.ppc
    for (x, y, z) in cells:
        acc = np.zeros((g.nv, 12), np.float32)
        aabs = np.zeros((g.nv, 12), np.float64)
        for k, sp in enumerate(wl.species):
            p0 = state["parts"][k]
            sel = []
            for dz in (-1, 0, 1):
                for dy in (-1, 0, 1):
                    for dx in (-1, 0, 1):
                        cx, cy, cz = [(c - 1 + d) % 128 for c, d in ((x, dx), (y, dy), (z, dz))]
                        cell = cx + 128 * (cy + 128 * cz)   # quiet start: cell-major, ppc per cell
                        sel.append(np.arange(cell * ppc, (cell + 1) * ppc))
            ps = p0[np.concatenate(sel)].copy()
            orc.advance_p(g, sp.q, sp.m, ps, interp_o, acc, aabs)
        v = g.voxel(x, y, z)
        got = acc_gpu[v].cpu().numpy()[None]
        assert_acc_close(got, acc[v][None], aabs[v][None])


def _ranks_from_standard(keys_std):
    """r of each standard-order position: position minus the first position of its key."""
    n = keys_std.numel()
    pos = torch.arange(n, device=keys_std.device)
    start = torch.ones(n, dtype=torch.bool, device=keys_std.device)
    start[1:] = keys_std[1:] != keys_std[:-1]
    first = torch.where(start, pos, torch.zeros_like(pos))
    first = torch.cummax(first, 0).values
    return pos - first


@pytest.mark.parametrize("order", [1, 2, 0])
def test_fullsize_sort_properties(state, order):
    vpic, g, hp = state["vpic"], state["g"], state["hp"]
    s = hp.species[0]                       # electrons after one push (no longer sorted)
    n = s.np
    p_in = s.p[:n]
    keys_in = p_in[:, 3].contiguous().view(torch.int32).long()
    out = torch.empty_like(p_in)
    perm = torch.empty(n, dtype=torch.int64, device="cuda")
    counts = torch.empty(g.nv, dtype=torch.int32, device="cuda")
    T = hp.ctx.info()["tile_sz"]
    ws = torch.empty(vpic.vpic_sort_workspace_bytes(hp.ctx, n, order), dtype=torch.uint8, device="cuda")
    vpic.vpic_sort_particles(hp.ctx, p_in, out, n, order, 0, ws, counts, None, perm)
    del ws
    torch.cuda.synchronize()
    # a permutation, payload moved with it, counts consistent
    assert torch.equal(torch.sort(perm).values, torch.arange(n, device="cuda"))
    assert torch.equal(out, p_in[perm])
    assert torch.equal(counts.long(), torch.bincount(keys_in, minlength=g.nv))
    k = keys_in[perm]
    # rank of each input particle among equal keys, in input order
    std = torch.sort(keys_in, stable=True).indices
    r_in = torch.empty(n, dtype=torch.int64, device="cuda")
    r_in[std] = _ranks_from_standard(keys_in[std])
    r = r_in[perm]
    if order == 0:
        tup = [k, perm]
    elif order == 1:
        tup = [r, k]
    else:
        tup = [k // T, r, k]
    # strictly increasing lexicographic tuples
    gt = torch.zeros(n - 1, dtype=torch.bool, device="cuda")
    eq = torch.ones(n - 1, dtype=torch.bool, device="cuda")
    for c in tup:
        gt |= eq & (c[1:] > c[:-1])
        eq &= c[1:] == c[:-1]
    assert bool(gt.all())


def test_fullsize_rho_total_charge(state):
    """vpic_accumulate_rho on the advanced configs[1] species (the bench's
    launch configuration; f4 diagnostic): total node charge = q sum w (closed
    form, conserved by the periodic step) and the mean node charge = one
    cell's worth."""
    V, hp, g = state["vpic"], state["hp"], state["g"]
    for k, sp in enumerate(state["wl"].species):
        s = hp.species[k]
        rho = torch.zeros(g.nv, dtype=torch.float32, device="cuda")
        V.vpic_accumulate_rho(hp.ctx, sp.q, s.p, s.np, rho)
        tot = float(np.float32(sp.q)) * state["parts"][k]["w"].astype(np.float64).sum()
        assert abs(rho.double().sum().item() - tot) < 1e-5 * abs(tot)
        node = rho[torch.from_numpy(g.interior_voxels()).cuda()].double()
        assert abs(node.mean().item() - tot / g.ncells) < 1e-5 * abs(tot / g.ncells)


def _record_multiset_hash(p: torch.Tensor, n: int) -> tuple:
    """Order-independent fingerprint of n 32-B records on the device: the sum
    and the xor of a 64-bit mix of each record (two independent folds), plus
    n.  Equal multisets give equal fingerprints; a lost, duplicated or altered
    record changes both folds with overwhelming probability."""
    w = p[:n].contiguous().view(torch.int64)              # [n, 4] words
    m = torch.tensor([0x9E3779B97F4A7C15 - (1 << 64), 0xC2B2AE3D27D4EB4F - (1 << 64),
                      0x165667B19E3779F9, 0x27D4EB2F165667C5], dtype=torch.int64, device=p.device)
    h = (w * m).sum(1)
    h = h ^ (h >> 29)
    h = h * (0xBF58476D1CE4E5B9 - (1 << 64))
    h = h ^ (h >> 32)
    x = h.clone()
    while x.numel() > 1:                                   # xor-fold
        if x.numel() & 1:
            x = torch.cat([x, torch.zeros(1, dtype=x.dtype, device=x.device)])
        x = x[0::2] ^ x[1::2]
    return n, int(h.sum().item()), int(x.item())


@pytest.mark.parametrize("device_exchange", [False, True], ids=["nccl", "device"])
def test_fullsize_loopback_single_round_matches_local(orc, device_exchange):
    """The multi-GPU exchange at full size (configs[1], 2^29 particles), in the
    configuration bench.py uses when there is an exchange: every periodic face
    routed through the single-round migration with a self peer (loopback).
    One IEEE-math PIC step must give exactly the particles of the local
    periodic wrap (as a multiset: fingerprints of all 2^29 records equal) and
    jf within the reordering tolerance."""
    from paper_conf_sc_tanlta25_b200 import vpic
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    wl = inputs.config(1)
    g = wl.grid
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, wl.field_amp, kind=wl.kind)
    out = []
    for loop in (False, True):
        hp = HotPath(wl, parts, fields, math=vpic.MATH_IEEE, loopback_exchange=loop,
                     device_exchange=loop and device_exchange, single_round=loop,
                     capacity_factor=1.01)
        hp.step(do_sort=True)
        torch.cuda.synchronize()
        fp = [_record_multiset_hash(s.p, s.np) for s in hp.species]
        jf = hp.jf.cpu().numpy()
        tail = hp.species[0].p[hp.species[0].np - 4096:hp.species[0].np].cpu()
        out.append((fp, jf, tail))
        hp.close()
        del hp
        torch.cuda.empty_cache()
    (fa, ja, ta), (fb, jb, tb) = out
    assert fa == fb
    assert not torch.equal(ta, tb)      # migration ran: arrivals were appended at the end
    # jf against the ORACLE on sampled edges (corners and faces of the box, where
    # the exchange and the ghost-accumulator reduction act, and random ones):
    # recomputed from every particle that can reach the 4 accumulators of each
    # edge (the 5^3 cells around it, periodic), per edge within T1
    rng = np.random.default_rng(3)
    cells = [(1, 1, 1), (128, 128, 128), (1, 64, 128), (128, 1, 64), (64, 128, 1)] + \
            [tuple(int(c) for c in rng.integers(1, 129, 3)) for _ in range(3)]
    interp_o = orc.load_interpolator(g, fields.copy())
    for (x, y, z) in cells:
        acc = np.zeros((g.nv, 12), np.float32)
        aabs = np.zeros((g.nv, 12), np.float64)
        for k, sp in enumerate(wl.species):
            sel = []
            for dz in range(-2, 3):
                for dy in range(-2, 3):
                    for dx in range(-2, 3):
                        cx, cy, cz = [(c - 1 + d) % 128 for c, d in ((x, dx), (y, dy), (z, dz))]
                        cell = cx + 128 * (cy + 128 * cz)   # quiet start: cell-major, ppc per cell
                        sel.append(np.arange(cell * wl.ppc, (cell + 1) * wl.ppc))
            ps = parts[k][np.concatenate(sel)].copy()
            orc.advance_p(g, sp.q, sp.m, ps, interp_o, acc, aabs)
        jo = orc.unload_accumulator(g, acc)
        jabs = orc.unload_accumulator(g, aabs.astype(np.float32)).astype(np.float64)
        v = g.voxel(x, y, z)
        for jg in (ja, jb):
            err = np.abs(jg[v, :3].astype(np.float64) - jo[v, :3])
            assert (err <= 1e-5 * jabs[v, :3] + 1e-30).all(), ((x, y, z), err, jabs[v, :3])

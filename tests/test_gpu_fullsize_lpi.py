"""Parity at full size for BASELINE.json configs[4] on ONE GPU -- the
laser-plasma slab, 512x256x256 cells, 64 ppc/species in the slab x in
[128, 384): 2 x 2^30 = 2^31 particles (68.7 GB), hot electrons drifting in
+x (u_th 0.2, drift 0.3: ~15% cross a face per step), cold heavy ions, static
laser E_y = cB_z -- in the launch configuration bench.py --config 4 times
(FAST math, AUTO deposit, TMA kernel).  The largest resident problem: 26-bit
voxel keys (4 radix passes), 2^30 records per species, byte offsets past
2^32.  One PIC step without the sort, so GPU particle i is input particle i:

* particles: 2^16 sampled per species, recomputed one by one by the oracle;
* accumulators: voxels on both slab edges and inside, recomputed by the
  oracle from every particle that starts in the 3x3x3 block around them;
* the standard-order sort of the advanced electrons (no perm output, to stay
  within HBM): keys non-decreasing, counts = histogram of the input keys,
  and the records a permutation of the input (two 64-bit multiset hashes).
"""
import numpy as np
import pytest
import torch

from paper_conf_sc_tanlta25_b200 import inputs
from parity_util import (assert_acc_close, assert_particles_bitexact, assert_particles_close, kick_bound,
                         replay_inputs, u_of)

pytestmark = pytest.mark.gpu

CH = 1 << 24   # rows per chunk of the device-side checks (small temporaries: ~161 GB resident)


@pytest.fixture(scope="module")
def lpi(orc):
    from paper_conf_sc_tanlta25_b200 import _build, vpic
    from paper_conf_sc_tanlta25_b200.pic import HotPath
    _build.build()
    wl = inputs.config(4)
    g = wl.grid
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, wl.field_amp, kind="lpi")
    hp = HotPath(wl, parts, fields, order=vpic.VPIC_SORT_STANDARD, math=vpic.MATH_FAST,
                 deposit=vpic.DEP_AUTO)
    hp.step(do_sort=False)
    torch.cuda.synchronize()
    interp_o = orc.load_interpolator(g, fields.copy())
    yield dict(wl=wl, g=g, parts=parts, hp=hp, interp_o=interp_o, vpic=vpic)
    hp.close()
    del hp
    torch.cuda.empty_cache()


def test_lpi_fullsize_particles_sampled(orc, lpi):
    wl, g, hp, interp_o = lpi["wl"], lpi["g"], lpi["hp"], lpi["interp_o"]
    rng = np.random.default_rng(5)
    for k, sp in enumerate(wl.species):
        p0 = lpi["parts"][k]
        assert p0.size == 1 << 30
        assert hp.species[k].np == p0.size          # periodic box: nobody leaves
        idx = np.sort(rng.choice(p0.size, 1 << 16, replace=False))
        idx[-1] = p0.size - 1                       # the last record (byte offset ~2^35)
        got = lpi["vpic"].particles_to_host(hp.species[k].p[torch.from_numpy(idx).cuda()])
        ps = p0[idx].copy()
        acc = np.zeros((g.nv, 12), np.float32)
        orc.advance_p(g, sp.q, sp.m, ps, interp_o, acc)
        assert_particles_close(g, got, ps, u_of(p0[idx]), kick_bound(g, p0[idx], sp.q, sp.m, interp_o))
        # T3: the move is the oracle's given the pushed momenta, bit for bit
        pr = replay_inputs(orc, g, sp.q, p0[idx].copy(), got)
        orc.move_deposit(g, sp.q, pr, None)
        assert_particles_bitexact(got, pr)


def test_lpi_fullsize_accumulator_sampled(orc, lpi):
    wl, g, hp, interp_o = lpi["wl"], lpi["g"], lpi["hp"], lpi["interp_o"]
    rng = np.random.default_rng(6)
    # slab edges (its first and last columns x = 129 / 384, and x = 385 that
    # only the +x-drifting electrons reach), the periodic y/z corners, and
    # random interior cells of the slab
    cells = [(129, 1, 1), (129, 256, 128), (384, 100, 256), (385, 7, 50)]
    cells += [(int(rng.integers(129, 385)), int(rng.integers(1, 257)), int(rng.integers(1, 257)))
              for _ in range(2)]
    for (x, y, z) in cells:
        block = np.array([g.voxel((x - 1 + dx) % g.nx + 1, (y - 1 + dy) % g.ny + 1, (z - 1 + dz) % g.nz + 1)
                          for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)], np.int32)
        acc = np.zeros((g.nv, 12), np.float32)
        aabs = np.zeros((g.nv, 12), np.float64)
        for k, sp in enumerate(wl.species):
            p0 = lpi["parts"][k]
            ps = p0[np.isin(p0["i"], block)].copy()
            orc.advance_p(g, sp.q, sp.m, ps, interp_o, acc, aabs)
        v = g.voxel(x, y, z)
        got = hp.acc[v].cpu().numpy()[None]
        assert aabs[v].sum() > 0
        assert_acc_close(got, acc[v][None], aabs[v][None])


def _multiset_hash(rows):
    """Two order-independent 64-bit hashes of int32 rows [n, 8] (chunked)."""
    mul = torch.tensor([0x9E3779B1, 0x85EBCA77, 0xC2B2AE3D, 0x27D4EB2F, 0x165667B1, 0xD3A2646C,
                        0xFD7046C5, 0xB55A4F09], dtype=torch.int64, device=rows.device)
    h1 = torch.zeros((), dtype=torch.int64, device=rows.device)
    h2 = torch.zeros((), dtype=torch.int64, device=rows.device)
    for a in range(0, rows.shape[0], CH):
        r = rows[a:a + CH].long() & 0xFFFFFFFF
        x = (r * mul).sum(1)
        x = x ^ (x >> 29)
        h1 += x.sum()
        h2 += ((x * 0x2545F4914F6CDD1D) ^ (x >> 17)).sum()
    return int(h1), int(h2)


def test_lpi_fullsize_sort_standard(lpi):
    vpic, g, hp = lpi["vpic"], lpi["g"], lpi["hp"]
    s = hp.species[0]                       # electrons after one push (no longer sorted)
    n = s.np
    p_in = s.p[:n]
    out = s.scratch[:n]
    counts = torch.empty(g.nv, dtype=torch.int32, device="cuda")
    vpic.vpic_sort_particles(hp.ctx, p_in, out, n, vpic.VPIC_SORT_STANDARD, 0, hp.ws, counts, None, None)
    torch.cuda.synchronize()
    kin = p_in.view(torch.int32)
    kout = out.view(torch.int32)
    hist = torch.zeros(g.nv, dtype=torch.int64, device="cuda")
    prev = torch.tensor(-1, dtype=torch.int32, device="cuda")
    for a in range(0, n, CH):
        hist += torch.bincount(kin[a:a + CH, 3].long(), minlength=g.nv)
        ko = kout[a:a + CH, 3]
        assert bool((ko[1:] >= ko[:-1]).all()) and bool(ko[0] >= prev)
        prev = ko[-1]
    assert torch.equal(counts.long(), hist)
    assert _multiset_hash(kout[:n]) == _multiset_hash(kin[:n])

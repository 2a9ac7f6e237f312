"""Seeded synthetic inputs shared by the tests, the bench and smoke().

This module holds NO arithmetic of the method (no push, sort, deposit or
interpolation): only the data layout (particle record, grid description) and
the seeded generators of the workloads named in BASELINE.json ``configs``
(recipes: DESIGN.md "Input recipe", after SURVEY.md §8(d)).

RNG: numpy's counter-based Philox4x32-10, key = (seed, species, chunk), so a
chunk's draws do not depend on how many threads generate the others.
"""
from __future__ import annotations

import math
import os
from concurrent.futures import ThreadPoolExecutor
from dataclasses import dataclass, field, replace
from typing import List, Sequence, Tuple

import numpy as np

PARTICLE_DTYPE = np.dtype(
    [("dx", "<f4"), ("dy", "<f4"), ("dz", "<f4"), ("i", "<i4"),
     ("ux", "<f4"), ("uy", "<f4"), ("uz", "<f4"), ("w", "<f4")])
assert PARTICLE_DTYPE.itemsize == 32

BC_PERIODIC, BC_REFLECT, BC_ABSORB = 0, 1, 2
SORT_STANDARD, SORT_STRIDED, SORT_TILED, SORT_NONE = 0, 1, 2, 3
ORDER_NAMES = {SORT_STANDARD: "standard", SORT_STRIDED: "strided",
               SORT_TILED: "tiled_strided", SORT_NONE: "none"}

MASTER_SEED = 0x5C2025
DT_COURANT = 0.95 / math.sqrt(3.0)   # c = dx = 1 units
_CHUNK = 1 << 22


@dataclass
class GridSpec:
    """Local block of a (possibly decomposed) periodic box.  Faces are
    ordered -x,-y,-z,+x,+y,+z; nbr_rank[f] == rank means a local wrap."""
    nx: int
    ny: int
    nz: int
    dx: float = 1.0
    dy: float = 1.0
    dz: float = 1.0
    dt: float = DT_COURANT
    cvac: float = 1.0
    pbc: Tuple[int, ...] = (0, 0, 0, 0, 0, 0)
    nbr_rank: Tuple[int, ...] = (0, 0, 0, 0, 0, 0)
    rank: int = 0
    gx0: int = 0
    gy0: int = 0
    gz0: int = 0
    gnx: int = 0        # global box width along x (0: this block is the whole box)

    @property
    def nv(self) -> int:
        return (self.nx + 2) * (self.ny + 2) * (self.nz + 2)

    @property
    def ncells(self) -> int:
        return self.nx * self.ny * self.nz

    def voxel(self, x, y, z):
        return x + (self.nx + 2) * (y + (self.ny + 2) * z)

    def coords(self, v):
        v = np.asarray(v, dtype=np.int64)
        sx, sy = self.nx + 2, self.ny + 2
        return v % sx, (v // sx) % sy, v // (sx * sy)

    def interior_voxels(self) -> np.ndarray:
        z, y, x = np.meshgrid(np.arange(1, self.nz + 1), np.arange(1, self.ny + 1),
                              np.arange(1, self.nx + 1), indexing="ij")
        return self.voxel(x, y, z).reshape(-1).astype(np.int32)


@dataclass
class Species:
    name: str
    q: float
    m: float
    u_th: float
    drift: Tuple[float, float, float] = (0.0, 0.0, 0.0)


@dataclass
class Workload:
    name: str
    grid: GridSpec
    species: List[Species]
    ppc: int                       # per species, mean
    steps: int
    sort_every: int
    kind: str = "uniform"          # uniform | harris | lpi
    field_amp: float = 0.01
    notes: str = ""


def config(idx: int) -> Workload:
    """BASELINE.json configs[idx] as a concrete single-GPU workload."""
    e = lambda: Species("electron", -1.0, 1.0, 0.1)
    if idx == 0:
        return Workload("uniform16_ppc32", GridSpec(16, 16, 16),
                        [e(), Species("ion", 1.0, 25.0, 0.02)], 32, 10, 10)
    if idx == 1:
        return Workload("uniform128_ppc128_sort20", GridSpec(128, 128, 128),
                        [e(), Species("ion", 1.0, 25.0, 0.02)], 128, 100, 20)
    if idx == 2:
        g = GridSpec(256, 128, 128, pbc=(0, 0, BC_REFLECT, 0, 0, BC_REFLECT))
        return Workload("harris256x128x128_ppc100", g,
                        [Species("electron", -1.0, 1.0, 0.1, (0.0, -0.005, 0.0)),
                         Species("ion", 1.0, 25.0, 0.02, (0.0, 0.005, 0.0))],
                        100, 100, 20, kind="harris")
    if idx == 3:
        return replace(config(1), name="weak_uniform128_per_gpu")
    if idx == 4:
        return Workload("lpi_slab512x256x256_ppc64", GridSpec(512, 256, 256),
                        [Species("electron", -1.0, 1.0, 0.2, (0.3, 0.0, 0.0)),
                         Species("ion", 1.0, 1836.0, 0.002)], 64, 100, 20, kind="lpi")
    if idx == 5:
        # the paper's strong-scaling regime (Fig. 9/10,
        # sorting disabled, per-GPU grids shrinking into
        # the cache).  256x128x128 cells: interpolator + accumulator 628 MB >>
        # the 126 MB L2 on one GPU, 81 MB per GPU on 8 (2x2x2 blocks of
        # 128x64x64).  Random (shuffled) order, no sort.
        return Workload("f3_l2strong_uniform256x128x128_ppc32_nosort", GridSpec(256, 128, 128),
                        [e(), Species("ion", 1.0, 25.0, 0.02)], 32, 100, 20,
                        notes="order none + shuffled")
    raise IndexError(idx)


# ------------------------------------------------------------ generators --
def _philox(seed: int, species: int, chunk: int) -> np.random.Generator:
    return np.random.Generator(np.random.Philox(key=[(seed << 16) ^ species, chunk]))


def _threads() -> int:
    try:
        return max(1, min(32, len(os.sched_getaffinity(0))))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def _fill_chunks(n: int, fn):
    chunks = [(c, c * _CHUNK, min(n, (c + 1) * _CHUNK)) for c in range((n + _CHUNK - 1) // _CHUNK)]
    if len(chunks) <= 1:
        for c in chunks:
            fn(*c)
        return
    with ThreadPoolExecutor(_threads()) as ex:
        list(ex.map(lambda c: fn(*c), chunks))


def particles_in_cells(cell_vox: np.ndarray, sp: Species, seed: int, sp_index: int,
                       weight: float) -> np.ndarray:
    """One particle per entry of cell_vox (already cell-major): offsets
    U(-1,1), momenta drift + u_th N(0,1) per component."""
    n = int(cell_vox.size)
    p = np.empty(n, PARTICLE_DTYPE)

    def fill(c, a, b):
        rng = _philox(seed, sp_index, c)
        m = b - a
        off = rng.random((3, m), dtype=np.float32)
        p["dx"][a:b] = off[0] * 2 - 1
        p["dy"][a:b] = off[1] * 2 - 1
        p["dz"][a:b] = off[2] * 2 - 1
        u = rng.standard_normal((3, m), dtype=np.float32)
        p["ux"][a:b] = u[0] * np.float32(sp.u_th) + np.float32(sp.drift[0])
        p["uy"][a:b] = u[1] * np.float32(sp.u_th) + np.float32(sp.drift[1])
        p["uz"][a:b] = u[2] * np.float32(sp.u_th) + np.float32(sp.drift[2])
        p["i"][a:b] = cell_vox[a:b]
        p["w"][a:b] = np.float32(weight)

    _fill_chunks(n, fill)
    return p


def uniform_cells(g: GridSpec, ppc: int) -> np.ndarray:
    return np.repeat(g.interior_voxels(), ppc)


def harris_cells(g: GridSpec, ppc_mean: int, seed: int, sp_index: int) -> np.ndarray:
    """Harris sheet n(z) = n_b + n_0 sech^2((z - zc)/L), n_b/n_0 = 0.2,
    L = 8 cells, mean ppc_mean per cell; sheet particles placed by the inverse
    CDF z = zc + L atanh(2U-1).  Returns cell-major voxel keys."""
    L, zc = 8.0, g.nz / 2.0
    total = ppc_mean * g.ncells
    # sheet fraction: n_0 * 2L / (n_b nz + n_0 2L) with n_b = 0.2 n_0
    sheet_frac = (2 * L) / (0.2 * g.nz + 2 * L)
    n_sheet = int(round(total * sheet_frac))
    rng = _philox(seed, 100 + sp_index, 0)
    u = rng.random(n_sheet)
    zs = zc + L * np.arctanh(np.clip(2 * u - 1, -1 + 1e-12, 1 - 1e-12))
    zs = np.clip(np.floor(zs).astype(np.int64), 0, g.nz - 1)
    xs = rng.integers(0, g.nx, n_sheet)
    ys = rng.integers(0, g.ny, n_sheet)
    nb = total - n_sheet
    xb = rng.integers(0, g.nx, nb)
    yb = rng.integers(0, g.ny, nb)
    zb = rng.integers(0, g.nz, nb)
    x = np.concatenate([xs, xb]) + 1
    y = np.concatenate([ys, yb]) + 1
    z = np.concatenate([zs, zb]) + 1
    v = g.voxel(x, y, z).astype(np.int32)
    v.sort(kind="stable")
    return v


def lpi_cells(g: GridSpec, ppc: int) -> np.ndarray:
    """Plasma slab x in [G/4, 3G/4) of the global box (G = g.gnx, or g.nx
    for an undecomposed box), ppc per slab cell: this block's part of it
    (global cell gx0 + x - 1 is local interior column x)."""
    G = g.gnx or g.nx
    x0 = max(G // 4 - g.gx0, 0)
    x1 = min(3 * G // 4 - g.gx0, g.nx)
    z, y, x = np.meshgrid(np.arange(1, g.nz + 1), np.arange(1, g.ny + 1),
                          np.arange(x0 + 1, max(x1, x0) + 1), indexing="ij")
    return np.repeat(g.voxel(x, y, z).reshape(-1).astype(np.int32), ppc)


def make_species_particles(wl: Workload, seed: int = None) -> List[np.ndarray]:
    seed = MASTER_SEED if seed is None else seed
    out = []
    for s, sp in enumerate(wl.species):
        if wl.kind == "harris":
            cells = harris_cells(wl.grid, wl.ppc, seed, s)
        elif wl.kind == "lpi":
            cells = lpi_cells(wl.grid, wl.ppc)
        else:
            cells = uniform_cells(wl.grid, wl.ppc)
        out.append(particles_in_cells(cells, sp, seed, s, 1.0 / wl.ppc))
    return out


def make_fields(g: GridSpec, amp: float = 0.01, seed: int = None, kind: str = "uniform") -> np.ndarray:
    """fields[nv][8] = ex,ey,ez,0,cbx,cby,cbz,0 (float32) over every voxel,
    ghosts included.  uniform: U(-amp, amp) noise.  harris: cbx = 0.5
    tanh((z - zc)/L) + noise.  lpi: ey = cbz = 0.02 sin(2 pi x / 32)."""
    seed = MASTER_SEED if seed is None else seed
    rng = _philox(seed, 999, 0)
    f = np.zeros((g.nv, 8), np.float32)
    noise = (rng.random((g.nv, 6), dtype=np.float32) * 2 - 1) * np.float32(amp)
    f[:, [0, 1, 2, 4, 5, 6]] = noise
    if kind in ("harris", "lpi"):
        x, y, z = g.coords(np.arange(g.nv))
        if kind == "harris":
            f[:, 4] += (0.5 * np.tanh((z - 0.5 - g.nz / 2.0) / 8.0)).astype(np.float32)
        else:
            s = (0.02 * np.sin(2 * np.pi * (x + g.gx0) / 32.0)).astype(np.float32)
            f[:, 1] += s
            f[:, 6] += s
    return f


def shuffle(p: np.ndarray, seed: int) -> np.ndarray:
    """The paper's 'random' order (Fig. 7): a seeded permutation."""
    rng = _philox(seed, 7777, 0)
    return p[rng.permutation(p.size)]


def random_particles(g: GridSpec, n: int, seed: int, u_scale: float = 0.5,
                     vox: Sequence[int] = None) -> np.ndarray:
    """Unstructured particles (random interior voxel, offsets, momenta) for
    edge-case parity tests."""
    rng = _philox(seed, 4242, 0)
    p = np.empty(n, PARTICLE_DTYPE)
    iv = g.interior_voxels() if vox is None else np.asarray(vox, np.int32)
    p["i"] = iv[rng.integers(0, iv.size, n)]
    for k in ("dx", "dy", "dz"):
        p[k] = (rng.random(n, dtype=np.float32) * 2 - 1)
    for k in ("ux", "uy", "uz"):
        p[k] = rng.standard_normal(n, dtype=np.float32) * np.float32(u_scale)
    p["w"] = rng.random(n, dtype=np.float32) + np.float32(0.5)
    return p


# ------------------------------------------------------- decomposition --
PROCESS_GRIDS = {1: (1, 1, 1), 2: (2, 1, 1), 4: (2, 2, 1), 8: (2, 2, 2)}


def process_grid(nranks: int) -> Tuple[int, int, int]:
    if nranks in PROCESS_GRIDS:
        return PROCESS_GRIDS[nranks]
    return (nranks, 1, 1)


def decompose(block: GridSpec, nranks: int, rank: int) -> GridSpec:
    """Rank `rank`'s block of a periodic box tiled by `block`-sized blocks on
    the process grid of `nranks` (x fastest).  PERIODIC faces point at the
    neighbour rank (a local wrap when the process grid is 1 wide there)."""
    P = process_grid(nranks)
    c = (rank % P[0], (rank // P[0]) % P[1], rank // (P[0] * P[1]))

    def rank_of(cc):
        cc = [cc[a] % P[a] for a in range(3)]
        return cc[0] + P[0] * (cc[1] + P[1] * cc[2])

    nbr, pbc = [], []
    for f in range(6):
        a = f % 3
        d = -1 if f < 3 else 1
        cc = list(c)
        cc[a] += d
        nbr.append(rank_of(cc))
        # the box's own wall (reflect / absorb) only on its outer faces; faces
        # between blocks are periodic (remote)
        outer = cc[a] < 0 or cc[a] >= P[a]
        pbc.append(block.pbc[f] if outer else BC_PERIODIC)
    n = (block.nx, block.ny, block.nz)
    return replace(block, nbr_rank=tuple(nbr), pbc=tuple(pbc), rank=rank,
                   gx0=c[0] * n[0], gy0=c[1] * n[1], gz0=c[2] * n[2])


def strong_decompose(box: GridSpec, nranks: int, rank: int) -> GridSpec:
    """Rank `rank`'s block when the periodic box `box` is SPLIT over the
    process grid of `nranks` (strong scaling: fixed global size, configs[4]);
    every dimension must divide."""
    P = process_grid(nranks)
    n = (box.nx, box.ny, box.nz)
    if any(n[a] % P[a] for a in range(3)):
        raise ValueError(f"{n} cells do not split over the process grid {P}")
    block = replace(box, nx=box.nx // P[0], ny=box.ny // P[1], nz=box.nz // P[2],
                    gnx=box.gnx or box.nx)
    return decompose(block, nranks, rank)


# ------------------------------------------------ block <-> global views --
def _block_coords(gg: GridSpec, gb: GridSpec, X, Y, Z):
    """Global interior cell coordinates -> block-local ones (may fall outside)."""
    return X - gb.gx0, Y - gb.gy0, Z - gb.gz0


def to_block(gg: GridSpec, gb: GridSpec, p: np.ndarray) -> np.ndarray:
    """The particles of the global box gg (voxels indexed on gg) that lie in
    block gb (a decompose()/strong_decompose() block of gg), re-indexed on gb."""
    X, Y, Z = gg.coords(p["i"])
    x, y, z = _block_coords(gg, gb, X, Y, Z)
    m = (x >= 1) & (x <= gb.nx) & (y >= 1) & (y <= gb.ny) & (z >= 1) & (z <= gb.nz)
    out = p[m].copy()
    out["i"] = gb.voxel(x[m], y[m], z[m]).astype(np.int32)
    return out


def to_global(gg: GridSpec, gb: GridSpec, p: np.ndarray) -> np.ndarray:
    """Block-indexed particles back on the global box's voxel indices."""
    x, y, z = gb.coords(p["i"])
    out = p.copy()
    out["i"] = gg.voxel(x + gb.gx0, y + gb.gy0, z + gb.gz0).astype(np.int32)
    return out


def block_fields(gg: GridSpec, gb: GridSpec, f: np.ndarray) -> np.ndarray:
    """fields[nv_block][8] of block gb cut from the global fields: interior
    and ghost voxels at the same global coordinates (a block's ghost plane is
    the neighbour block's interior plane, or the global box's own ghost plane
    on an outer face -- which a wall's caller-owned ghost values need)."""
    v = np.arange(gb.nv)
    x, y, z = gb.coords(v)
    return f[gg.voxel(x + gb.gx0, y + gb.gy0, z + gb.gz0)].copy()


def block_interior_to_global(gg: GridSpec, gb: GridSpec) -> Tuple[np.ndarray, np.ndarray]:
    """(block voxel, global voxel) index pairs of the block's interior."""
    vb = gb.interior_voxels().astype(np.int64)
    x, y, z = gb.coords(vb)
    return vb, gg.voxel(x + gb.gx0, y + gb.gy0, z + gb.gz0).astype(np.int64)

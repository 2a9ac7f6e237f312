"""TEST INFRASTRUCTURE ONLY -- ctypes wrapper of the serial C++ oracle.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  The product path
(``paper_conf_sc_tanlta25_b200``) never imports it; the two share no code.

The oracle follows PAPER.md (Alg. 1, Alg. 2, the push's
"gather phase, atomic scatter phase" P:238) and the VPIC reading of SURVEY.md
§8(c) for every formula the paper does not print; see ``vpic_oracle.cpp``.
Parity status of each function is listed in DESIGN.md ("Oracle pins").
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "vpic_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")

PARTICLE_DTYPE = np.dtype(
    [("dx", "<f4"), ("dy", "<f4"), ("dz", "<f4"), ("i", "<i4"),
     ("ux", "<f4"), ("uy", "<f4"), ("uz", "<f4"), ("w", "<f4")])
MOVER_DTYPE = np.dtype([("dispx", "<f4"), ("dispy", "<f4"), ("dispz", "<f4"), ("idx", "<i4")])

SORT_STANDARD, SORT_STRIDED, SORT_TILED, SORT_NONE = 0, 1, 2, 3


class OrcGrid(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nz", ctypes.c_int32),
                ("dx", ctypes.c_float), ("dy", ctypes.c_float), ("dz", ctypes.c_float),
                ("dt", ctypes.c_float), ("cvac", ctypes.c_float),
                ("pbc", ctypes.c_int32 * 6), ("nbr_rank", ctypes.c_int32 * 6),
                ("rank", ctypes.c_int32)]


def build(force: bool = False) -> str:
    """Compile liboracle.so (g++ -O2 -ffp-contract=off: no FMA contraction;
    -fopenmp for the all-core baseline orc_advance_p_omp only).
    ORACLE_LIB (dev: tools/oracle_mutations.py) names a prebuilt library to
    load instead -- a deliberately broken oracle the pins must reject."""
    if os.environ.get("ORACLE_LIB"):
        return os.environ["ORACLE_LIB"]
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "vpic_oracle.h"))):
        cmd = ["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
               "-fPIC", "-shared", _SRC, "-o", _LIB + ".tmp"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        G = ctypes.POINTER(OrcGrid)
        _lib.orc_sort_keys.argtypes = [P, I64, ctypes.c_int, I64, P, P]
        _lib.orc_sort_keys.restype = ctypes.c_int
        _lib.orc_sort_particles.argtypes = [G, P, P, I64, ctypes.c_int, I64, P, P, P]
        _lib.orc_sort_particles.restype = ctypes.c_int
        _lib.orc_load_interpolator.argtypes = [G, P, P]
        _lib.orc_load_interpolator.restype = None
        _lib.orc_advance_p.argtypes = [G, ctypes.c_float, ctypes.c_float, P, I64, P, P, P, P, P, I64]
        _lib.orc_advance_p.restype = I64
        _lib.orc_advance_p_omp.argtypes = [G, ctypes.c_float, ctypes.c_float, P, I64, P, P, P, I64,
                                           ctypes.c_int]
        _lib.orc_advance_p_omp.restype = I64
        _lib.orc_continuity_residual.argtypes = [G, P, P, P, P, P]
        _lib.orc_continuity_residual.restype = None
        _lib.orc_move_deposit.argtypes = [G, ctypes.c_float, P, I64, P, P, P, P, I64]
        _lib.orc_move_deposit.restype = I64
        _lib.orc_move_p.argtypes = [G, P, P, P, P, P, ctypes.c_float]
        _lib.orc_move_p.restype = ctypes.c_int
        _lib.orc_unload_accumulator.argtypes = [G, P, P]
        _lib.orc_unload_accumulator.restype = None
        _lib.orc_unload_raw.argtypes = [G, P, P]
        _lib.orc_unload_raw.restype = None
        _lib.orc_accumulate_rho.argtypes = [G, P, I64, ctypes.c_float, P]
        _lib.orc_accumulate_rho.restype = None
        _lib.orc_remove_absorbed.argtypes = [G, P, I64, P, I64]
        _lib.orc_remove_absorbed.restype = I64
        _lib.orc_advance_b.argtypes = [G, P, ctypes.c_float]
        _lib.orc_advance_b.restype = None
        _lib.orc_advance_e.argtypes = [G, P, P, ctypes.c_float]
        _lib.orc_advance_e.restype = None
        _lib.orc_gather_scatter.argtypes = [P, P, I64, P, P, P, I64, I64]
        _lib.orc_gather_scatter.restype = None
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def make_grid(spec) -> OrcGrid:
    """Marshal an ``inputs.GridSpec`` (or any object with the same fields)."""
    g = OrcGrid()
    g.nx, g.ny, g.nz = spec.nx, spec.ny, spec.nz
    g.dx, g.dy, g.dz, g.dt, g.cvac = spec.dx, spec.dy, spec.dz, spec.dt, spec.cvac
    for f in range(6):
        g.pbc[f] = spec.pbc[f]
        g.nbr_rank[f] = spec.nbr_rank[f]
    g.rank = spec.rank
    return g


def nvox(spec) -> int:
    return (spec.nx + 2) * (spec.ny + 2) * (spec.nz + 2)


# ------------------------------------------------------------------ sort --
def sort_keys(keys, order, tile_sz=1):
    keys = np.ascontiguousarray(keys, dtype=np.int32)
    n = keys.size
    nk = np.empty(n, np.int64)
    perm = np.empty(n, np.int64)
    rc = lib().orc_sort_keys(_ptr(keys), n, order, tile_sz, _ptr(nk), _ptr(perm))
    if rc:
        raise ValueError("orc_sort_keys rejected its arguments")
    return nk, perm


def sort_particles(spec, p, order, tile_sz=1):
    """Returns (sorted particles, voxel counts[nv], new_keys[np], perm[np])."""
    p = np.ascontiguousarray(p, dtype=PARTICLE_DTYPE)
    out = np.empty_like(p)
    counts = np.empty(nvox(spec), np.int32)
    nk = np.empty(p.size, np.int64)
    perm = np.empty(p.size, np.int64)
    g = make_grid(spec)
    rc = lib().orc_sort_particles(ctypes.byref(g), _ptr(p), _ptr(out), p.size, order, tile_sz,
                                  _ptr(counts), _ptr(nk), _ptr(perm))
    if rc:
        raise ValueError("orc_sort_particles rejected its arguments")
    return out, counts, nk, perm


# ------------------------------------------------------------ push path --
def load_interpolator(spec, fields):
    """fields: float32[nv, 8] (ghost planes filled in place). Returns interp[nv, 20]."""
    assert fields.dtype == np.float32 and fields.flags.c_contiguous
    interp = np.empty((nvox(spec), 20), np.float32)
    g = make_grid(spec)
    lib().orc_load_interpolator(ctypes.byref(g), _ptr(fields), _ptr(interp))
    return interp


def advance_p(spec, q, m, p, interp, acc, acc_abs=None, max_movers=None, acc_cond=None):
    """In place on p (PARTICLE_DTYPE) and acc (float32[nv,12]). Returns movers.
    acc_abs / acc_cond (float64[nv,12], optional): sum of |contribution| and
    of |q uX| per entry (tolerances T1 / T3)."""
    assert p.dtype == PARTICLE_DTYPE and p.flags.c_contiguous
    assert acc.dtype == np.float32 and acc.flags.c_contiguous
    if max_movers is None:
        max_movers = p.size
    movers = np.zeros(max(max_movers, 1), MOVER_DTYPE)
    g = make_grid(spec)
    nm = lib().orc_advance_p(ctypes.byref(g), q, m, _ptr(p), p.size, _ptr(interp), _ptr(acc),
                             _ptr(acc_abs), _ptr(acc_cond), _ptr(movers), max_movers)
    if nm < 0:
        raise OverflowError("mover list overflow")
    return movers[:nm].copy()


def advance_p_omp(spec, q, m, p, interp, acc, threads, max_movers=None):
    """advance_p over `threads` particle blocks (OpenMP, private accumulators)."""
    assert p.dtype == PARTICLE_DTYPE and p.flags.c_contiguous
    assert acc.dtype == np.float32 and acc.flags.c_contiguous
    if max_movers is None:
        max_movers = p.size
    movers = np.zeros(max(max_movers, 1), MOVER_DTYPE)
    g = make_grid(spec)
    nm = lib().orc_advance_p_omp(ctypes.byref(g), q, m, _ptr(p), p.size, _ptr(interp), _ptr(acc),
                                 _ptr(movers), max_movers, int(threads))
    if nm < 0:
        raise OverflowError("mover list overflow")
    return movers[:nm].copy()


def move_deposit(spec, q, p, acc, acc_abs=None, max_movers=None):
    """The move + deposit half of advance_p on particles whose momenta are
    already pushed (in place on p and acc).  Returns movers."""
    assert p.dtype == PARTICLE_DTYPE and p.flags.c_contiguous
    assert acc is None or (acc.dtype == np.float32 and acc.flags.c_contiguous)
    if max_movers is None:
        max_movers = p.size
    movers = np.zeros(max(max_movers, 1), MOVER_DTYPE)
    g = make_grid(spec)
    nm = lib().orc_move_deposit(ctypes.byref(g), q, _ptr(p), p.size, _ptr(acc), _ptr(acc_abs), None,
                                _ptr(movers), max_movers)
    if nm < 0:
        raise OverflowError("mover list overflow")
    return movers[:nm].copy()


def move_p(spec, p1, mover, acc, qsp, acc_abs=None, acc_cond=None):
    """move_p on a single particle record (np.void / 1-element array) in place."""
    g = make_grid(spec)
    return lib().orc_move_p(ctypes.byref(g), _ptr(p1), _ptr(mover), _ptr(acc), _ptr(acc_abs),
                            _ptr(acc_cond), qsp)


def unload_accumulator(spec, acc):
    jf = np.empty((nvox(spec), 4), np.float32)
    g = make_grid(spec)
    lib().orc_unload_accumulator(ctypes.byref(g), _ptr(np.ascontiguousarray(acc)), _ptr(jf))
    return jf


def unload_raw(spec, acc):
    J = np.empty((nvox(spec), 4), np.float64)
    g = make_grid(spec)
    lib().orc_unload_raw(ctypes.byref(g), _ptr(np.ascontiguousarray(acc)), _ptr(J))
    return J


def accumulate_rho(spec, p, q, rho=None):
    if rho is None:
        rho = np.zeros(nvox(spec), np.float64)
    g = make_grid(spec)
    p = np.ascontiguousarray(p, dtype=PARTICLE_DTYPE)
    lib().orc_accumulate_rho(ctypes.byref(g), _ptr(p), p.size, q, _ptr(rho))
    return rho


def continuity_residual(spec, rho0, rho1, jf):
    """(res, mag) per node, float64[nv] (NaN outside the node range): the
    discrete continuity residual of float32 rho0/rho1[nv], jf[nv,4] (D1)."""
    rho0 = np.ascontiguousarray(rho0, np.float32)
    rho1 = np.ascontiguousarray(rho1, np.float32)
    jf = np.ascontiguousarray(jf, np.float32)
    res = np.full(rho0.size, np.nan)
    mag = np.full(rho0.size, np.nan)
    g = make_grid(spec)
    lib().orc_continuity_residual(ctypes.byref(g), _ptr(rho0), _ptr(rho1), _ptr(jf), _ptr(res), _ptr(mag))
    return res, mag


def remove_absorbed(spec, p, movers):
    g = make_grid(spec)
    n = lib().orc_remove_absorbed(ctypes.byref(g), _ptr(p), p.size, _ptr(movers), movers.size)
    return p[:n].copy()


# ------------------------------------------------------------ field solver --
def advance_b(spec, fields, frac):
    """In place on fields float32[nv, 8] (ghost planes refreshed)."""
    assert fields.dtype == np.float32 and fields.flags.c_contiguous
    g = make_grid(spec)
    lib().orc_advance_b(ctypes.byref(g), _ptr(fields), frac)


def advance_e(spec, fields, jf, eps0=1.0):
    assert fields.dtype == np.float32 and fields.flags.c_contiguous
    jf = np.ascontiguousarray(jf, dtype=np.float32)
    g = make_grid(spec)
    lib().orc_advance_e(ctypes.byref(g), _ptr(fields), _ptr(jf), eps0)


# ------------------------------------------------------ gather-scatter (f2) --
def gather_scatter(keys, x, table, acc, stencil_nx=0):
    """Returns out[n]; acc (float64[nkeys]) updated in place."""
    keys = np.ascontiguousarray(keys, dtype=np.int32)
    x = np.ascontiguousarray(x, dtype=np.float64)
    table = np.ascontiguousarray(table, dtype=np.float64)
    out = np.empty(keys.size, np.float64)
    lib().orc_gather_scatter(_ptr(keys), _ptr(x), keys.size, _ptr(table), _ptr(out), _ptr(acc),
                             table.size, stencil_nx)
    return out

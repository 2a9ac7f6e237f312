"""Thin ctypes binding of libvpic.so (include/vpic.h): argument marshalling only.

Every function has the C name and forwards torch CUDA tensors as raw device
pointers plus the current CUDA stream.  Nothing here computes any part of the
method; if libvpic.so is missing or no sm_100 device is present, the calls
raise -- there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import torch

from .inputs import GridSpec

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("VPIC_LIB") or os.path.join(_HERE, "libvpic.so")  # VPIC_LIB: dev A/B builds

VPIC_OK, VPIC_ERR_INVALID, VPIC_ERR_CAPACITY = 0, -1, -2
VPIC_ERR_CUDA, VPIC_ERR_NCCL, VPIC_ERR_UNSUPPORTED = -3, -4, -5
VPIC_SORT_STANDARD, VPIC_SORT_STRIDED, VPIC_SORT_TILED_STRIDED, VPIC_SORT_NONE = 0, 1, 2, 3
VPIC_OPT_MATH, VPIC_OPT_DEPOSIT, VPIC_OPT_TILE_SZ, VPIC_OPT_ADVANCE_KERNEL = 0, 1, 2, 3
VPIC_OPT_LOOPBACK_EXCHANGE = 4
VPIC_OPT_ADVANCE_CTAS_PER_SM = 5
VPIC_OPT_DEVICE_EXCHANGE = 6
VPIC_OPT_SINGLE_ROUND_MIGRATION = 7
MATH_FAST, MATH_IEEE = 0, 1
DEP_AUTO, DEP_LANE, DEP_WARP, DEP_SMEM = 0, 1, 2, 3

# every symbol include/vpic.h declares (checked by tests/test_abi_symbols.py)
EXPORTS = ["vpic_get_unique_id", "vpic_ctx_create", "vpic_ctx_destroy", "vpic_ctx_set_option",
           "vpic_ctx_info", "vpic_status_string", "vpic_sort_workspace_bytes",
           "vpic_sort_particles", "vpic_load_interpolator", "vpic_clear_accumulator",
           "vpic_advance_p", "vpic_advance_p_dev", "vpic_unload_accumulator", "vpic_migrate_particles", "vpic_migrate_particles_dev",
           "vpic_kernel_launches", "vpic_advance_b", "vpic_advance_e", "vpic_gather_scatter",
           "vpic_accumulate_rho", "vpic_continuity_residual", "vpic_run_host_workspace_bytes",
           "vpic_run_host", "vpic_sort_particles_keyed", "vpic_advance_p_keys"]


class VpicError(RuntimeError):
    def __init__(self, fn, status):
        self.status = status
        msg = _lib.vpic_status_string(status).decode() if _lib is not None else str(status)
        super().__init__(f"{fn} failed: {msg} ({status})")


class vpic_grid_t(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nz", ctypes.c_int32),
                ("dx", ctypes.c_float), ("dy", ctypes.c_float), ("dz", ctypes.c_float),
                ("dt", ctypes.c_float), ("cvac", ctypes.c_float),
                ("pbc", ctypes.c_int32 * 6), ("nbr_rank", ctypes.c_int32 * 6),
                ("gx0", ctypes.c_int32), ("gy0", ctypes.c_int32), ("gz0", ctypes.c_int32)]


_lib: Optional[ctypes.CDLL] = None


def load(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libvpic.so (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(f"libvpic.so not built ({path}); run __graft_entry__.build()")
    lib = ctypes.CDLL(path)
    P, I64, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
    sig = {
        "vpic_get_unique_id": ([P], I),
        "vpic_ctx_create": ([ctypes.POINTER(P), ctypes.POINTER(vpic_grid_t), I, I, P, I], I),
        "vpic_ctx_destroy": ([P], I),
        "vpic_ctx_set_option": ([P, I, I64], I),
        "vpic_ctx_info": ([P, P], I),
        "vpic_status_string": ([I], ctypes.c_char_p),
        "vpic_kernel_launches": ([], I64),
        "vpic_sort_workspace_bytes": ([P, I64, I], ctypes.c_size_t),
        "vpic_sort_particles": ([P, P, P, I64, I, I64, P, ctypes.c_size_t, P, P, P, P], I),
        "vpic_load_interpolator": ([P, P, P, P], I),
        "vpic_clear_accumulator": ([P, P, P], I),
        "vpic_advance_p": ([P, ctypes.c_float, ctypes.c_float, P, I64, P, P, P, I64, P, P, P], I),
        "vpic_unload_accumulator": ([P, P, P, P], I),
        "vpic_advance_b": ([P, P, ctypes.c_float, P], I),
        "vpic_gather_scatter": ([P, P, P, I64, P, P, P, I64, I64, I, P], I),
        "vpic_accumulate_rho": ([P, ctypes.c_float, P, I64, P, P], I),
        "vpic_continuity_residual": ([P, P, P, P, P, P, P], I),
        "vpic_advance_e": ([P, P, P, ctypes.c_float, P], I),
        "vpic_migrate_particles": ([P, ctypes.c_float, ctypes.c_float, P, ctypes.POINTER(I64),
                                    I64, P, I64, P, P, P], I),
        "vpic_advance_p_dev": ([P, ctypes.c_float, ctypes.c_float, P, P, I64, P, P, P, I64, P, P, P], I),
        "vpic_migrate_particles_dev": ([P, ctypes.c_float, ctypes.c_float, P, P, I64, P, I64, P, P, P, P], I),
        "vpic_run_host_workspace_bytes": ([P, I, P, I], ctypes.c_size_t),
        "vpic_sort_particles_keyed": ([P, P, P, I64, I, I64, P, P, ctypes.c_size_t, P, P, P, P], I),
        "vpic_advance_p_keys": ([P, ctypes.c_float, ctypes.c_float, P, I64, P, P, P, I64, P, P, P, P], I),
        "vpic_run_host": ([P, I, P, P, P, I, I64, I, I, P, I, ctypes.c_float, P, ctypes.c_size_t,
                           ctypes.POINTER(I64), P], I),
    }
    for name, (args, res) in sig.items():
        if os.environ.get("VPIC_LIB") and not hasattr(lib, name):
            continue   # dev A/B against an older build: newer entry points absent
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    _lib = lib
    return lib


def _ptr(t) -> Optional[int]:
    if t is None:
        return None
    if isinstance(t, int):
        return t
    if isinstance(t, torch.Tensor):
        if not t.is_cuda:
            raise ValueError("libvpic takes device tensors only")
        if not t.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return t.data_ptr()
    raise TypeError(type(t))


def _stream(stream) -> Optional[int]:
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


def _check(fn, rc):
    if rc != VPIC_OK:
        raise VpicError(fn, rc)


def make_grid(spec: GridSpec) -> vpic_grid_t:
    g = vpic_grid_t()
    g.nx, g.ny, g.nz = spec.nx, spec.ny, spec.nz
    g.dx, g.dy, g.dz, g.dt, g.cvac = spec.dx, spec.dy, spec.dz, spec.dt, spec.cvac
    for f in range(6):
        g.pbc[f] = spec.pbc[f]
        g.nbr_rank[f] = spec.nbr_rank[f]
    g.gx0, g.gy0, g.gz0 = spec.gx0, spec.gy0, spec.gz0
    return g


# ------------------------------------------------------------------ API --
def vpic_get_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check("vpic_get_unique_id", load().vpic_get_unique_id(buf))
    return bytes(buf)


class Context:
    """Owns a vpic_ctx*; the methods are the C calls with the ctx bound."""

    def __init__(self, spec: GridSpec, rank: int = 0, nranks: int = 1, uid: bytes = None,
                 device: int = None):
        lib = load()
        if device is None:
            device = torch.cuda.current_device()
        self.spec = spec
        self.device = device
        self._g = make_grid(spec)
        h = ctypes.c_void_p()
        ub = None if uid is None else (ctypes.c_uint8 * 128).from_buffer_copy(uid)
        _check("vpic_ctx_create", lib.vpic_ctx_create(ctypes.byref(h), ctypes.byref(self._g), rank,
                                                      nranks, ub, device))
        self.h = h

    def close(self):
        if getattr(self, "h", None) and self.h.value:
            load().vpic_ctx_destroy(self.h)
            self.h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_option(self, option: int, value: int):
        _check("vpic_ctx_set_option", load().vpic_ctx_set_option(self.h, option, value))

    def info(self):
        a = (ctypes.c_int64 * 8)()
        _check("vpic_ctx_info", load().vpic_ctx_info(self.h, a))
        return dict(zip(["num_sms", "tile_sz", "nv", "rank", "nranks", "l2_bytes", "math",
                         "deposit"], list(a)))


def vpic_kernel_launches() -> int:
    return int(load().vpic_kernel_launches())


def vpic_sort_workspace_bytes(ctx: Context, np_: int, order: int) -> int:
    return int(load().vpic_sort_workspace_bytes(ctx.h, np_, order))


def vpic_sort_particles(ctx: Context, p_in, p_out, np_: int, order: int, tile_sz: int = 0,
                        ws=None, voxel_counts=None, new_keys=None, perm=None, stream=None):
    ws_bytes = 0 if ws is None else ws.numel() * ws.element_size()
    _check("vpic_sort_particles", load().vpic_sort_particles(
        ctx.h, _ptr(p_in), _ptr(p_out), np_, order, tile_sz, _ptr(ws), ws_bytes,
        _ptr(voxel_counts), _ptr(new_keys), _ptr(perm), _stream(stream)))


def vpic_sort_particles_keyed(ctx: Context, p_in, p_out, np_: int, order: int, tile_sz: int, keys,
                              ws=None, voxel_counts=None, new_keys=None, perm=None, stream=None):
    ws_bytes = 0 if ws is None else ws.numel() * ws.element_size()
    _check("vpic_sort_particles_keyed", load().vpic_sort_particles_keyed(
        ctx.h, _ptr(p_in), _ptr(p_out), np_, order, tile_sz, _ptr(keys), _ptr(ws), ws_bytes,
        _ptr(voxel_counts), _ptr(new_keys), _ptr(perm), _stream(stream)))


def vpic_advance_p_keys(ctx: Context, q: float, m: float, p, np_: int, interp, acc, movers=None,
                        max_movers: int = 0, n_movers=None, flags=None, keys_out=None, stream=None):
    _check("vpic_advance_p_keys", load().vpic_advance_p_keys(
        ctx.h, q, m, _ptr(p), np_, _ptr(interp), _ptr(acc), _ptr(movers), max_movers,
        _ptr(n_movers), _ptr(flags), _ptr(keys_out), _stream(stream)))


def vpic_load_interpolator(ctx: Context, fields, interp, stream=None):
    _check("vpic_load_interpolator",
           load().vpic_load_interpolator(ctx.h, _ptr(fields), _ptr(interp), _stream(stream)))


def vpic_clear_accumulator(ctx: Context, acc, stream=None):
    _check("vpic_clear_accumulator", load().vpic_clear_accumulator(ctx.h, _ptr(acc), _stream(stream)))


def vpic_advance_p(ctx: Context, q: float, m: float, p, np_: int, interp, acc, movers=None,
                   max_movers: int = 0, n_movers=None, flags=None, stream=None):
    _check("vpic_advance_p", load().vpic_advance_p(
        ctx.h, q, m, _ptr(p), np_, _ptr(interp), _ptr(acc), _ptr(movers), max_movers,
        _ptr(n_movers), _ptr(flags), _stream(stream)))


def vpic_unload_accumulator(ctx: Context, acc, jf, stream=None):
    _check("vpic_unload_accumulator",
           load().vpic_unload_accumulator(ctx.h, _ptr(acc), _ptr(jf), _stream(stream)))


def vpic_advance_b(ctx: Context, fields, frac: float, stream=None):
    _check("vpic_advance_b", load().vpic_advance_b(ctx.h, _ptr(fields), frac, _stream(stream)))


def vpic_advance_e(ctx: Context, fields, jf, eps0: float = 1.0, stream=None):
    _check("vpic_advance_e", load().vpic_advance_e(ctx.h, _ptr(fields), _ptr(jf), eps0,
                                                   _stream(stream)))


def vpic_gather_scatter(ctx: Context, keys, x, table, out, acc, stencil_nx: int = 0,
                        aggregate: int = 0, stream=None):
    _check("vpic_gather_scatter", load().vpic_gather_scatter(
        ctx.h, _ptr(keys), _ptr(x), keys.numel(), _ptr(table), _ptr(out), _ptr(acc), table.numel(),
        stencil_nx, aggregate, _stream(stream)))


def vpic_accumulate_rho(ctx: Context, q: float, p, np_: int, rho, stream=None):
    _check("vpic_accumulate_rho", load().vpic_accumulate_rho(ctx.h, q, _ptr(p), np_, _ptr(rho),
                                                             _stream(stream)))


def vpic_continuity_residual(ctx: Context, rho0, rho1, jf, out, res=None, stream=None):
    _check("vpic_continuity_residual", load().vpic_continuity_residual(
        ctx.h, _ptr(rho0), _ptr(rho1), _ptr(jf), _ptr(out), _ptr(res) if res is not None else None,
        _stream(stream)))


def vpic_migrate_particles(ctx: Context, q: float, m: float, p, np_: int, max_np: int, movers,
                           max_movers: int, n_movers, acc, stream=None) -> int:
    n = ctypes.c_int64(np_)
    _check("vpic_migrate_particles", load().vpic_migrate_particles(
        ctx.h, q, m, _ptr(p), ctypes.byref(n), max_np, _ptr(movers), max_movers, _ptr(n_movers),
        _ptr(acc), _stream(stream)))
    return int(n.value)


def vpic_advance_p_dev(ctx: Context, q: float, m: float, p, np_dev, max_np: int, interp, acc,
                       movers=None, max_movers: int = 0, n_movers=None, flags=None, stream=None):
    """vpic_advance_p with the particle count in device memory (int64[1])."""
    _check("vpic_advance_p_dev", load().vpic_advance_p_dev(
        ctx.h, q, m, _ptr(p), _ptr(np_dev), max_np, _ptr(interp), _ptr(acc), _ptr(movers), max_movers,
        _ptr(n_movers), _ptr(flags), _stream(stream)))


def vpic_migrate_particles_dev(ctx: Context, q: float, m: float, p, np_dev, max_np: int, movers,
                               max_movers: int, n_movers, acc, flags, stream=None):
    """vpic_migrate_particles with the count in device memory: no host
    synchronisation (single-round, device-initiated exchange only)."""
    _check("vpic_migrate_particles_dev", load().vpic_migrate_particles_dev(
        ctx.h, q, m, _ptr(p), _ptr(np_dev), max_np, _ptr(movers), max_movers, _ptr(n_movers),
        _ptr(acc), _ptr(flags), _stream(stream)))


# ------------------------------------------------------- tensor helpers --
def interp_coefficients(interp, nv: int):
    """The 18 interpolator coefficients per voxel, [nv][18] float32 in the
    order of include/vpic.h, from an interp[nv][24] buffer in the library's
    layout: nv rows of the first 16 coefficients (64 B), then nv pairs
    (cbz, dcbz/dz) (8 B each); the last nv x 24 B are unused."""
    import numpy as np
    a = np.ascontiguousarray(interp.detach().cpu().numpy() if hasattr(interp, "detach") else interp,
                             dtype=np.float32).reshape(-1)
    rows = a[:16 * nv].reshape(nv, 16)
    tail = a[16 * nv:18 * nv].reshape(nv, 2)
    return np.concatenate([rows, tail], axis=1)

class vpic_species_host_t(ctypes.Structure):
    _fields_ = [("q", ctypes.c_float), ("m", ctypes.c_float), ("host_in", ctypes.c_void_p),
                ("host_out", ctypes.c_void_p), ("np", ctypes.c_int64), ("max_np", ctypes.c_int64),
                ("dev", ctypes.c_void_p * 4)]


def _species_host(species):
    """[(q, m, host_in, host_out | None, np, [4 device buffers])] -> C array."""
    arr = (vpic_species_host_t * len(species))()
    for k, (q, m, hin, hout, n, dev) in enumerate(species):
        assert hin.is_pinned() and (hout is None or hout.is_pinned()), "host buffers must be pinned"
        arr[k].q, arr[k].m = q, m
        arr[k].host_in = hin.data_ptr()
        arr[k].host_out = hout.data_ptr() if hout is not None else None
        arr[k].np = n
        arr[k].max_np = min(b.shape[0] for b in dev)
        for b in range(4):
            arr[k].dev[b] = dev[b].data_ptr()
    return arr


def vpic_run_host_workspace_bytes(ctx: Context, species, order: int) -> int:
    arr = _species_host(species)
    return int(load().vpic_run_host_workspace_bytes(ctx.h, len(species), arr, order))


def vpic_run_host(ctx: Context, species, fields_host, jf_host, order: int, tile_sz: int, steps: int,
                  n_cycles: int, deposit_modes=None, field_solve: bool = False, eps0: float = 1.0,
                  ws=None, stream=None) -> int:
    """n_cycles sort periods from / to pinned host memory through the C ABI
    (copies pipelined inside the library); returns particles x PIC steps."""
    import numpy as np
    arr = _species_host(species)
    modes = None
    if deposit_modes is not None:
        modes = np.ascontiguousarray(deposit_modes, dtype=np.int8)
        assert modes.size == steps * len(species)
    pushes = ctypes.c_int64(0)
    ws_bytes = 0 if ws is None else ws.numel() * ws.element_size()
    _check("vpic_run_host", load().vpic_run_host(
        ctx.h, len(species), arr, fields_host.data_ptr(), jf_host.data_ptr(), order, tile_sz, steps,
        n_cycles, modes.ctypes.data if modes is not None else None, int(field_solve), eps0, _ptr(ws),
        ws_bytes, ctypes.byref(pushes), _stream(stream)))
    return int(pushes.value)


def particles_to_device(p_np, device="cuda") -> torch.Tensor:
    """Host structured particle array -> device float32 [n, 8] view (32 B records)."""
    import numpy as np
    t = torch.from_numpy(np.ascontiguousarray(p_np).view(np.float32).reshape(-1, 8))
    return t.to(device)


def particles_to_host(t: torch.Tensor):
    from .inputs import PARTICLE_DTYPE
    return t.detach().cpu().contiguous().numpy().view(PARTICLE_DTYPE).reshape(-1)

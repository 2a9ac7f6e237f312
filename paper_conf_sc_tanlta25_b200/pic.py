"""The hot path as a user drives it: device-resident state for one rank and a
PIC step made only of libvpic C-ABI calls:

    [every S steps] vpic_sort_particles (per species)
    vpic_load_interpolator -> vpic_clear_accumulator
    -> vpic_advance_p (per species) -> [vpic_migrate_particles]
    -> vpic_unload_accumulator
    [-> vpic_advance_b(1/2) -> vpic_advance_e -> vpic_advance_b(1/2)]   (field_solve)

PyTorch only provides device memory, pinned host memory and the stream.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Optional

import numpy as np
import torch

from . import inputs, vpic


def bind_to_gpu_cpus(device: int) -> Optional[int]:
    """Restrict this process to the CPUs NVML reports as local to `device`
    (its NUMA node), so pinned host buffers allocated afterwards are
    first-touched next to the GPU's PCIe root. Returns the number of CPUs
    bound to, or None when NVML cannot tell (nothing changed)."""
    import os
    try:
        import pynvml
        p = torch.cuda.get_device_properties(device)
        bus = "%08x:%02x:%02x.0" % (p.pci_domain_id, p.pci_bus_id, p.pci_device_id)
        pynvml.nvmlInit()
        try:
            h = pynvml.nvmlDeviceGetHandleByPciBusId(bus)
            ncpu = os.cpu_count() or 1
            words = pynvml.nvmlDeviceGetCpuAffinity(h, (ncpu + 63) // 64)
        finally:
            pynvml.nvmlShutdown()
    except Exception:
        return None
    local = {64 * w + b for w, m in enumerate(words) for b in range(64) if (int(m) >> b) & 1}
    cpus = local & os.sched_getaffinity(0)
    if not cpus:
        return None
    os.sched_setaffinity(0, cpus)
    return len(cpus)


@dataclass
class SpeciesState:
    name: str
    q: float
    m: float
    p: torch.Tensor          # [cap, 8] float32 (32-B records)
    scratch: torch.Tensor    # sort output buffer, same shape
    np: int
    movers: torch.Tensor     # [max_movers, 4]
    n_movers: torch.Tensor   # int64[1]
    flags: torch.Tensor      # int32[1]
    np_dev: torch.Tensor = None   # int64[1]: the count on the device (graph mode)
    keys: torch.Tensor = None     # uint32-as-int32 [cap]: voxels from the last advance (keyed sort)
    keys_valid: bool = False


# thermal spread (cells) since the sort within which DEP_SMEM pays (DESIGN.md
# §10): from 0.4 cell same-voxel groups are common enough to sum; past ~1.3
# cells (hot species late in the period) they are mostly singletons again
SMEM_SIGMA = 0.4
SMEM_SIGMA_MAX = 1.3


def auto_deposit_mode(u_th: float, cvac: float, dt: float, dmin: float, steps_since_sort: int) -> int:
    """The AUTO policy: the deposit mode for a species of thermal speed u_th,
    `steps_since_sort` PIC steps after its sort (cell size dmin)."""
    sigma = u_th * cvac * dt / dmin * steps_since_sort
    return vpic.DEP_SMEM if SMEM_SIGMA <= sigma < SMEM_SIGMA_MAX else vpic.DEP_WARP


class HotPath:
    def __init__(self, wl: inputs.Workload, species_particles: List[np.ndarray], fields: np.ndarray,
                 order: int = vpic.VPIC_SORT_STANDARD, math: int = vpic.MATH_FAST,
                 deposit: int = vpic.DEP_AUTO, tile_sz: int = 0, rank: int = 0, nranks: int = 1,
                 uid: bytes = None, capacity_factor: float = 1.0, max_movers: int = 1 << 20,
                 device: Optional[int] = None, field_solve: bool = False, eps0: float = 1.0,
                 loopback_exchange: bool = False, concurrent_species: bool = False,
                 device_exchange: bool = False, inbox_cap: int = 0, single_round: bool = False,
                 graphs: bool = False, keyed_sort: bool = True, device_exchange_fallback: bool = False):
        vpic.load()
        self.wl = wl
        self.g = wl.grid
        self.dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
        self.ctx = vpic.Context(self.g, rank, nranks, uid, self.dev.index)
        self.ctx.set_option(vpic.VPIC_OPT_MATH, math)
        # deposit AUTO: per species and step, SMEM (small same-voxel groups
        # summed in shared memory) while the species' thermal spread since its
        # sort (thermal speed x steps) is in [SMEM_SIGMA, SMEM_SIGMA_MAX),
        # WARP otherwise
        self.deposit_auto = deposit == vpic.DEP_AUTO
        self._dep_mode = vpic.DEP_WARP if self.deposit_auto else deposit
        self.ctx.set_option(vpic.VPIC_OPT_DEPOSIT, self._dep_mode)
        self.steps_since_sort = 0
        self.order = order
        self.tile_sz = tile_sz
        self.field_solve = field_solve   # advance_b(1/2), advance_e, advance_b(1/2) after unload
        self.eps0 = eps0
        self.nranks = nranks
        if loopback_exchange:   # periodic faces through the NCCL path (self peer)
            self.ctx.set_option(vpic.VPIC_OPT_LOOPBACK_EXCHANGE, 1)
        if single_round:        # moves finished in the ghost layer, one 26-neighbour exchange
            self.ctx.set_option(vpic.VPIC_OPT_SINGLE_ROUND_MIGRATION, 1)
        self.exchange_note = None
        if device_exchange:     # movers stored into the neighbours' inboxes by the push (f4)
            try:
                self.ctx.set_option(vpic.VPIC_OPT_DEVICE_EXCHANGE, inbox_cap if inbox_cap > 1 else 1)
            except vpic.VpicError as e:
                if not device_exchange_fallback:
                    raise
                # peers not load/store reachable (no NVLink / symmetric memory):
                # the NCCL send/recv exchange of the same migration mode
                device_exchange = False
                self.exchange_note = f"device-initiated exchange unavailable ({e}); NCCL send/recv used"
                import sys
                print(f"HotPath: {self.exchange_note}", file=sys.stderr, flush=True)
        self.device_exchange = device_exchange
        self.migrate = (nranks > 1 or loopback_exchange
                        or any(b == inputs.BC_ABSORB for b in self.g.pbc))
        # species pushed concurrently on their own streams, each persistent
        # kernel on one CTA slot of every SM (not with migration: its counts
        # synchronise per species)
        self.concurrent = concurrent_species and not self.migrate and len(wl.species) > 1
        if self.concurrent:
            self.ctx.set_option(vpic.VPIC_OPT_ADVANCE_CTAS_PER_SM, 1)
            self.sp_streams = [torch.cuda.Stream(device=self.dev) for _ in wl.species]
        nv = self.g.nv
        f32 = dict(dtype=torch.float32, device=self.dev)
        self.fields = torch.from_numpy(np.ascontiguousarray(fields)).to(self.dev)
        self.interp = torch.zeros((nv, 24), **f32)
        self.acc = torch.zeros((nv, 12), **f32)
        self.jf = torch.zeros((nv, 4), **f32)
        self.species: List[SpeciesState] = []
        max_np = 0
        for sp, ph in zip(wl.species, species_particles):
            n = int(ph.size)
            cap = max(1, int(n * capacity_factor))
            p = torch.empty((cap, 8), **f32)
            if n:
                p[:n].copy_(torch.from_numpy(np.ascontiguousarray(ph).view(np.float32).reshape(-1, 8)))
            self.species.append(SpeciesState(
                sp.name, sp.q, sp.m, p, torch.empty_like(p), n,
                torch.zeros((max_movers, 4), **f32),
                torch.zeros(1, dtype=torch.int64, device=self.dev),
                torch.zeros(1, dtype=torch.int32, device=self.dev)))
            max_np = max(max_np, cap)
        ws = vpic.vpic_sort_workspace_bytes(self.ctx, max_np, order)
        self.ws = torch.empty(max(ws, 1), dtype=torch.uint8, device=self.dev)
        # CUDA-graph mode: the PIC steps of a sort period are captured once per
        # particle-buffer configuration and replayed; particle counts live on
        # the device (vpic_advance_p_dev / vpic_migrate_particles_dev: no host
        # synchronisation inside a period).  Needs no migration, or the
        # single-round device-initiated exchange.
        self.graphs = graphs
        self.keyed_sort = keyed_sort    # the period's last push writes the next sort's keys
        if graphs:
            if self.migrate and not (single_round and device_exchange):
                raise ValueError("graphs need the single-round device-initiated exchange (or none)")
            if self.concurrent:
                raise ValueError("graphs and concurrent species are exclusive")
            for sp in self.species:
                sp.np_dev = torch.tensor([sp.np], dtype=torch.int64, device=self.dev)
        self._graphs = {}
        self._warm = False
        self._host_bufs = None  # run_host_cycles: the 4 device buffers per species
        self._host_ws = None
        self.adv_events = []   # (start, end) CUDA events around advance_p, when recording
        self.sort_events = []  # (start, end, species) around vpic_sort_particles
        self.record_advance = False

    def _set_deposit(self, k: int):
        """AUTO deposit policy for species k at the current step."""
        if not self.deposit_auto:
            return
        g = self.g
        mode = auto_deposit_mode(self.wl.species[k].u_th, g.cvac, g.dt, min(g.dx, g.dy, g.dz),
                                 self.steps_since_sort)
        if mode != self._dep_mode:
            self.ctx.set_option(vpic.VPIC_OPT_DEPOSIT, mode)
            self._dep_mode = mode

    # ------------------------------------------------------------ calls --
    @property
    def n_particles(self) -> int:
        return sum(s.np for s in self.species)

    def sort(self, order: Optional[int] = None):
        order = self.order if order is None else order
        if order == vpic.VPIC_SORT_NONE:
            return
        stream = torch.cuda.current_stream()
        for s in self.species:
            if self.record_advance:
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
            if s.keys_valid:   # keys written by the period's last advance_p
                vpic.vpic_sort_particles_keyed(self.ctx, s.p, s.scratch, s.np, order, self.tile_sz, s.keys,
                                               self.ws)
            else:
                vpic.vpic_sort_particles(self.ctx, s.p, s.scratch, s.np, order, self.tile_sz, self.ws)
            s.keys_valid = False
            if self.record_advance:
                e1.record(stream)
                self.sort_events.append((e0, e1, s.name))
            s.p, s.scratch = s.scratch, s.p
        self.steps_since_sort = 0

    def step(self, do_sort: bool = False, emit_keys: bool = False):
        """One PIC step.  emit_keys: the last step of a sort period -- the
        push also writes every particle's voxel for the next sort
        (vpic_advance_p_keys + vpic_sort_particles_keyed: no pass over the
        records to read the keys), when nothing migrates."""
        if do_sort:
            self.sort()
        keyed = emit_keys and self.keyed_sort and not self.migrate and not self.concurrent
        vpic.vpic_load_interpolator(self.ctx, self.fields, self.interp)
        vpic.vpic_clear_accumulator(self.ctx, self.acc)
        stream = torch.cuda.current_stream()
        if self.concurrent:
            ready = torch.cuda.Event()
            ready.record(stream)
            for k, (s, st) in enumerate(zip(self.species, self.sp_streams)):
                self._set_deposit(k)
                st.wait_event(ready)
                if self.record_advance:
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(st)
                vpic.vpic_advance_p(self.ctx, s.q, s.m, s.p, s.np, self.interp, self.acc, s.movers,
                                    s.movers.shape[0], s.n_movers, s.flags, stream=st)
                s.keys_valid = False
                if self.record_advance:
                    e1.record(st)
                    self.adv_events.append((e0, e1, s.np))
            for st in self.sp_streams:
                stream.wait_stream(st)
        for k, s in enumerate(() if self.concurrent else self.species):
            self._set_deposit(k)
            if self.record_advance:
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
            if keyed:
                if s.keys is None:
                    s.keys = torch.empty(s.p.shape[0], dtype=torch.int32, device=self.dev)
                vpic.vpic_advance_p_keys(self.ctx, s.q, s.m, s.p, s.np, self.interp, self.acc, s.movers,
                                         s.movers.shape[0], s.n_movers, s.flags, s.keys)
            else:
                vpic.vpic_advance_p(self.ctx, s.q, s.m, s.p, s.np, self.interp, self.acc, s.movers,
                                    s.movers.shape[0], s.n_movers, s.flags)
            s.keys_valid = keyed
            if self.record_advance:
                e1.record(stream)
                self.adv_events.append((e0, e1, s.np))
            if self.migrate:
                # VPIC_ERR_CAPACITY (raised) if advance_p dropped movers
                s.np = vpic.vpic_migrate_particles(self.ctx, s.q, s.m, s.p, s.np, s.p.shape[0],
                                                   s.movers, s.movers.shape[0], s.n_movers, self.acc)
                fl = int(s.flags.item())      # (the stream is synchronised by the migration)
                if fl:
                    raise vpic.VpicError(f"advance_p ({s.name}: flags {fl:#x})", vpic.VPIC_ERR_CAPACITY)
                s.n_movers.zero_()
        vpic.vpic_unload_accumulator(self.ctx, self.acc, self.jf)
        if self.field_solve:
            vpic.vpic_advance_b(self.ctx, self.fields, 0.5)
            vpic.vpic_advance_e(self.ctx, self.fields, self.jf, self.eps0)
            vpic.vpic_advance_b(self.ctx, self.fields, 0.5)
        self.steps_since_sort += 1

    def cycle(self, steps: int):
        """One sort period: sort, then `steps` PIC steps."""
        if self.graphs:
            return self._cycle_graph(steps)
        for k in range(steps):
            self.step(do_sort=(k == 0), emit_keys=(k == steps - 1))

    # ------------------------------------------------------- graph mode --
    def sync_counts(self):
        """Graph mode: bring the device particle counts (and capacity flags)
        back to the host."""
        if not self.graphs:
            return
        torch.cuda.current_stream().synchronize()
        for s in self.species:
            s.np = int(s.np_dev.item())
            fl = int(s.flags.item())
            if fl:
                raise vpic.VpicError(f"graph-mode step ({s.name}: flags {fl:#x})", vpic.VPIC_ERR_CAPACITY)

    def _step_dev(self):
        vpic.vpic_load_interpolator(self.ctx, self.fields, self.interp)
        vpic.vpic_clear_accumulator(self.ctx, self.acc)
        for k, s in enumerate(self.species):
            self._set_deposit(k)
            vpic.vpic_advance_p_dev(self.ctx, s.q, s.m, s.p, s.np_dev, s.p.shape[0], self.interp, self.acc,
                                    s.movers, s.movers.shape[0], s.n_movers, s.flags)
            s.keys_valid = False
            if self.migrate:
                vpic.vpic_migrate_particles_dev(self.ctx, s.q, s.m, s.p, s.np_dev, s.p.shape[0], s.movers,
                                                s.movers.shape[0], s.n_movers, self.acc, s.flags)
                s.n_movers.zero_()
        vpic.vpic_unload_accumulator(self.ctx, self.acc, self.jf)
        if self.field_solve:
            vpic.vpic_advance_b(self.ctx, self.fields, 0.5)
            vpic.vpic_advance_e(self.ctx, self.fields, self.jf, self.eps0)
            vpic.vpic_advance_b(self.ctx, self.fields, 0.5)
        self.steps_since_sort += 1

    def _cycle_graph(self, steps: int):
        self.sync_counts()
        self.sort()
        for s in self.species:
            s.np_dev.fill_(s.np)
        if self.migrate and (steps * len(self.species)) % 2:
            for _ in range(steps):     # (an odd number of exchanges cannot be replayed)
                self._step_dev()
            return
        key = (steps, tuple(s.p.data_ptr() for s in self.species), self.fields.data_ptr())
        if not self._warm:             # first period eagerly: lazy allocations, attributes
            for _ in range(steps):
                self._step_dev()
            self._warm = True
            return
        gr = self._graphs.get(key)
        if gr is None:
            torch.cuda.synchronize()
            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr):
                for _ in range(steps):
                    self._step_dev()
            self._graphs[key] = gr
        gr.replay()

    # ------------------------------------------------------- host <-> device --
    def run_host_cycles(self, host_in, host_out, fields_host, jf_host, n_cycles: int, S: int):
        """Stream `n_cycles` sort periods from pinned host memory through the
        C ABI's host-buffer driver (vpic_run_host): every cycle uploads its
        particle and field inputs and downloads jf and, unless host_out is
        None, its particles; the library overlaps cycle k+1's upload and
        cycle k-1's download with cycle k's compute (4 device particle
        buffers per species rotate).  The deposit mode per species and step
        is this HotPath's (AUTO policy or fixed).  Returns the pushes done
        (particles x PIC steps)."""
        if self._host_bufs is None:
            self._host_bufs = [[s.p, s.scratch, torch.empty_like(s.p), torch.empty_like(s.p)]
                               for s in self.species]
        species = [(s.q, s.m, host_in[j], None if host_out is None else host_out[j], host_in[j].shape[0],
                    self._host_bufs[j]) for j, s in enumerate(self.species)]
        modes = np.empty((S, len(self.species)), np.int8)
        for t in range(S):
            for j, sp in enumerate(self.wl.species):
                modes[t, j] = (auto_deposit_mode(sp.u_th, self.g.cvac, self.g.dt,
                                                 min(self.g.dx, self.g.dy, self.g.dz), t)
                               if self.deposit_auto else self._dep_mode)
        need = vpic.vpic_run_host_workspace_bytes(self.ctx, species, self.order)
        if self._host_ws is None or self._host_ws.numel() < need:
            self._host_ws = torch.empty(need, dtype=torch.uint8, device=self.dev)
        pushes = vpic.vpic_run_host(self.ctx, species, fields_host, jf_host, self.order, self.tile_sz, S,
                                    n_cycles, modes, self.field_solve, self.eps0, self._host_ws)
        for j, s in enumerate(self.species):
            s.np = host_in[j].shape[0]
            s.keys_valid = False
        return pushes

    def particles_host(self, k: int) -> np.ndarray:
        self.sync_counts()
        s = self.species[k]
        return vpic.particles_to_host(s.p[:s.np])

    def close(self):
        torch.cuda.synchronize()
        self._graphs.clear()        # captured graphs reference the context's NCCL state
        self.ctx.close()

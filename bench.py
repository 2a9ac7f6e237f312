#!/usr/bin/env python
"""Benchmark of the VPIC particle hot path on B200 (BASELINE.json metric:
particle pushes/sec (advance_p + sort) per GPU and at N GPUs; % of HBM roofline).

One bench step = one sort period of the workload: vpic_sort_particles (per
species) followed by S = sort_every PIC steps of load_interpolator ->
clear_accumulator -> advance_p (per species) [-> migrate] ->
unload_accumulator, all through the C-ABI on device-resident inputs
(BASELINE.json configs[1]: uniform 128^3, 128 ppc/species, sort every 20).
value = pushes (particles x PIC steps, all ranks) / max-over-ranks device time.

    python bench.py [--gpus N --steps K --warmup W]           # our arm
    python bench.py --impl reference [...]                    # the oracle on host cores
N > 1: launch with torch.distributed.run (one rank per GPU, NCCL); the box is
weak-scaled (a 128^3 block per GPU, BASELINE.json configs[3]).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

FALLBACK_HBM_GBS = 6650.0
# VPIC_BENCH_SHARE_GPU=1 (test of the N > 1 code path on a 1-GPU box, not a
# measurement): every rank on GPU 0, torch.distributed over gloo, and the
# library's NCCL communicator over sockets (each rank poses as its own host)
SHARE_GPU = os.environ.get("VPIC_BENCH_SHARE_GPU") == "1"
METRIC = "particle pushes/sec (advance_p+sort)"
UNIT = "pushes/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=1,
                    help="BASELINE.json configs[] index (0-4); 5 = SURVEY §8(f) f3: L2-resident strong "
                         "scaling, 256x128x128 uniform, 32 ppc, random order, sorting off")
    ap.add_argument("--block-of", type=int, default=1,
                    help="1 GPU: run rank 0's block of the config's box split over this many ranks "
                         "(locally periodic; the compute side of a strong-scaling point)")
    ap.add_argument("--order", default=None, choices=["standard", "strided", "tiled_strided", "none"],
                    help="sort order (default: standard; none for --config 5)")
    ap.add_argument("--shuffle", action="store_true", help="random initial order (paper's 'random'; "
                                                           "default for --config 5)")
    ap.add_argument("--sort-every", type=int, default=0)
    ap.add_argument("--math", default="fast", choices=["fast", "ieee"])
    ap.add_argument("--deposit", default="auto", choices=["auto", "lane", "warp", "smem"])
    ap.add_argument("--kernel", default="auto", choices=["auto", "direct", "tma"])
    ap.add_argument("--field-solve", action="store_true",
                    help="full PIC step: + advance_b/advance_e (self-consistent fields)")
    ap.add_argument("--concurrent-species", action="store_true",
                    help="push the species concurrently on two streams (1 CTA/SM each)")
    ap.add_argument("--exchange", default="auto", choices=["auto", "nccl", "device"],
                    help="particle exchange when there is one (N>1 or --loopback): device-initiated "
                         "(symmetric-memory inboxes, the default) or NCCL send/recv rounds")
    ap.add_argument("--migration", default="auto", choices=["auto", "rounds", "single"],
                    help="with an exchange: single-round 26-neighbour migration (moves finished in "
                         "the ghost layer; the default) or up to 3 face rounds")
    ap.add_argument("--loopback", action="store_true",
                    help="1 GPU: periodic faces through the NCCL exchange (self peer)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no e2e/cpu legs)")
    a = ap.parse_args()
    if a.order is None:
        a.order = "none" if a.config == 5 else "standard"
    if a.config == 5:
        a.shuffle = True
    return a


ORDERS = {"standard": 0, "strided": 1, "tiled_strided": 2, "none": 3}


# ------------------------------------------------------------ helpers --
class ClockSampler:
    """nvidia-smi clocks / throttle reasons during the timed region."""

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 7:
                self.rows.append(parts)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows for k in range(4) if r[3 + k].lower() == "active"})
        load = [s for s in sm]
        return {"sm_mhz": statistics.median(load) if load else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons, "samples": len(self.rows)}


def hbm_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback"


def committed_traffic(kernel_key: str, workload: str):
    """dram bytes per launch of the dominant kernel from the committed ncu
    --set full summary (profiles/traffic.json), if it matches this workload."""
    path = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        with open(path) as f:
            t = json.load(f)
        e = t.get(kernel_key, {})
        if e.get("workload") == workload:
            return e.get("dram_bytes_per_launch"), e
    except Exception:
        pass
    return None, None


# --------------------------------------------------------- CPU / oracle --
def oracle_sample_workload(cfg: int = 1):
    """The reference arm's bounded sample: the same plasma recipe (species,
    ppc, u_th, fields, boundaries, sort period) as configs[cfg] on a small box
    (32x32x16 uniform; 32x16x32 Harris sheet; 64x16x16 LPI slab)."""
    from paper_conf_sc_tanlta25_b200 import inputs
    from dataclasses import replace
    wl = inputs.config(3 if cfg == 3 else cfg)
    n = {"uniform": (32, 32, 16), "harris": (32, 16, 32), "lpi": (64, 16, 16)}[wl.kind]
    if cfg == 5:
        n = (64, 32, 32)
    return replace(wl, grid=replace(wl.grid, nx=n[0], ny=n[1], nz=n[2]),
                   name=wl.name + "@%dx%dx%d" % n)


def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def cpu_model() -> str:
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.lower().startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def run_oracle_steps(wl, n_steps, sort_every, order, threads=1):
    """The oracle on the host: per step one sort of each species (serial)
    and sort_every PIC steps; the push on `threads` cores (orc_advance_p_omp:
    particle blocks with private accumulators) when threads > 1."""
    import oracle
    from paper_conf_sc_tanlta25_b200 import inputs
    oracle.build()
    g = wl.grid
    parts = inputs.make_species_particles(wl)
    fields = inputs.make_fields(g, wl.field_amp, kind=wl.kind)
    acc = np.zeros((g.nv, 12), np.float32)
    times = []
    pushes = 0
    for step in range(n_steps):
        t0 = time.perf_counter()
        for k in range(sort_every):
            if k == 0 and order != 3:
                parts = [oracle.sort_particles(g, p, order, 3 * 148 * 128)[0] for p in parts]
            interp = oracle.load_interpolator(g, fields)
            acc[:] = 0
            for sp, p in zip(wl.species, parts):
                if threads > 1:
                    oracle.advance_p_omp(g, sp.q, sp.m, p, interp, acc, threads)
                else:
                    oracle.advance_p(g, sp.q, sp.m, p, interp, acc)
                pushes += p.size
            oracle.unload_accumulator(g, acc)
        times.append(time.perf_counter() - t0)
    return times, sum(p.size for p in parts) * sort_every


STRONG_CONFIGS = (4, 5)


def effective_config(args, world):
    """The configs[] index a run measures: as given on one GPU; under torchrun
    the weak-scaling configs[3], or configs[4] / the f3 box split over the
    ranks (strong)."""
    return args.config if (world == 1 or args.config in STRONG_CONFIGS) else 3


def reference_arm(args, rank, world):
    if rank != 0:
        return
    from paper_conf_sc_tanlta25_b200 import inputs
    cfg = effective_config(args, world)
    wl = oracle_sample_workload(cfg)
    S = args.sort_every or wl.sort_every
    order = ORDERS[args.order]
    cores = host_cores()
    _ = run_oracle_steps(wl, max(args.warmup, 0) and 1, S, order, cores)  # untimed warm-up (1 step)
    times, per_step = run_oracle_steps(wl, args.steps, S, order, cores)
    total = sum(times)
    value = per_step * args.steps / total
    out = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total / args.steps,
        "higher_is_better": True, "scaling": "strong" if (world > 1 and cfg in STRONG_CONFIGS) else "weak",
        "vs_baseline": None, "dtype": "f32",
        "data": "synthetic",
        "config": {"workload": inputs.config(cfg).name, "order": args.order, "sort_every": S,
                   "sample": f"{wl.name}: {per_step // S} particles per step (bounded CPU sample)"},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "cpu_model": cpu_model(),
                         "sample": f"C++ oracle (oracle/; push on {cores} cores with OpenMP particle blocks "
                                   f"and private accumulators, sort serial), {wl.name}: {per_step // S} "
                                   f"particles, sort + {S} PIC steps per step"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(out), flush=True)


def cpu_baseline(args):
    """The oracle on this box's host cores (SURVEY.md §8(d) "Oracle timing"):
    (ii) all cores of the affinity mask (OpenMP particle blocks, private
    accumulators) -- the reported value -- and (i) one core, serial."""
    wl = oracle_sample_workload(args.config)
    S = args.sort_every or wl.sort_every
    cores = host_cores()
    t1, per_step = run_oracle_steps(wl, 1, S, ORDERS[args.order], 1)
    tn, _ = run_oracle_steps(wl, 4, S, ORDERS[args.order], cores)   # first period warms the threads
    one = per_step / t1[0]
    alln = 3 * per_step / sum(tn[1:])
    return {"value": alln, "unit": UNIT, "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
            "single_core": {"value": one, "unit": UNIT, "cores": 1},
            "per_core_all": alln / cores,
            "sample": f"C++ oracle on {wl.name} ({per_step // S} particles): one sort (serial) + {S} "
                      f"PIC steps; {sum(tn[1:]) / 3:.2f} s per period with the push on {cores} cores (OpenMP "
                      f"particle blocks, private accumulators; mean of 3 after a warm-up period), "
                      f"{t1[0]:.1f} s serial on 1 core"}


# ---------------------------------------------------------------- ours --
def our_arm(args, rank, world):
    import torch
    import torch.distributed as dist
    from paper_conf_sc_tanlta25_b200 import inputs, vpic
    from paper_conf_sc_tanlta25_b200.pic import HotPath

    from paper_conf_sc_tanlta25_b200.pic import bind_to_gpu_cpus
    local = 0 if SHARE_GPU else int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    red_dev = "cpu" if SHARE_GPU else dev   # gloo reduces host tensors
    # pinned e2e buffers first-touched on the GPU's NUMA node (2-socket nodes)
    cpu_bind = bind_to_gpu_cpus(local)
    # N > 1: weak scaling on configs[3] (C2 per GPU), or strong scaling of
    # the LPI slab (configs[4], --config 4: the 512x256x256 box split over
    # the process grid)
    strong = world > 1 and args.config in STRONG_CONFIGS
    wl = inputs.config(effective_config(args, world))
    S = args.sort_every or wl.sort_every
    order = ORDERS[args.order]
    box = wl.grid
    if strong:
        g = inputs.strong_decompose(wl.grid, world, rank)
    elif world == 1 and args.block_of > 1:
        # rank 0's block of a block_of-way split, its faces wrapped locally:
        # one strong-scaling point's per-GPU compute without the exchange
        g = inputs.strong_decompose(wl.grid, args.block_of, 0)
        g = replace_grid(g, nbr_rank=(0,) * 6, rank=0)
    else:
        g = inputs.decompose(wl.grid, world, rank) if world > 1 else wl.grid
    from dataclasses import replace
    wl = replace(wl, grid=g)
    uid = None
    if world > 1:
        obj = [vpic.vpic_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    seed = inputs.MASTER_SEED + 1 + rank
    parts = inputs.make_species_particles(wl, seed)
    if args.shuffle:
        parts = [inputs.shuffle(p, seed + 17 + k) for k, p in enumerate(parts)]
    fields = inputs.make_fields(g, wl.field_amp, seed, kind=wl.kind)
    math_mode = vpic.MATH_IEEE if args.math == "ieee" else vpic.MATH_FAST
    dep = {"auto": 0, "lane": 1, "warp": 2, "smem": 3}[args.deposit]
    # particle capacity per rank: the drifting LPI electrons pile up on the
    # downstream ranks (~0.13% of a rank's electrons cross each step at 2
    # GPUs); movers per inbox slot: a boundary plane's electrons x 0.35 (the
    # crossing fraction per step of a drift-0.3, u_th-0.2 population is ~0.17)
    cap = 1.0 if world == 1 else (1.5 if strong else 1.05)
    inbox = 0
    if strong:
        plane = max(g.ny * g.nz, g.nx * g.nz, g.nx * g.ny)
        inbox = max(1 << 19, int(0.35 * wl.ppc * plane))
    hp = HotPath(wl, parts, fields, order=order, math=math_mode, deposit=dep, rank=rank,
                 nranks=world, uid=uid, capacity_factor=cap, device=local, inbox_cap=inbox,
                 field_solve=args.field_solve, loopback_exchange=args.loopback and world == 1,
                 concurrent_species=args.concurrent_species,
                 device_exchange=args.exchange in ("auto", "device") and (world > 1 or args.loopback),
                 device_exchange_fallback=args.exchange == "auto",
                 single_round=args.migration in ("auto", "single") and (world > 1 or args.loopback))
    hp.ctx.set_option(vpic.VPIC_OPT_ADVANCE_KERNEL, {"auto": 0, "direct": 1, "tma": 2}[args.kernel])
    n_local = hp.n_particles
    comm = {"nranks": world, "vpic_ctx_nranks": int(hp.ctx.info()["nranks"]),
            "backend": dist.get_backend() if world > 1 else None}

    def barrier():
        if world > 1:
            dist.barrier()

    # ---- warm-up
    for _ in range(args.warmup):
        hp.cycle(S)
    torch.cuda.synchronize()
    barrier()

    # ---- timed region (device-resident inputs; 17 GB of particles >> 126 MB L2)
    stream = torch.cuda.current_stream()
    hp.adv_events = []
    hp.sort_events = []
    hp.record_advance = True
    launches0 = vpic.vpic_kernel_launches()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    pushes_local = 0
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        barrier()
        e0.record(stream)
        marks = [e0]
        for k in range(args.steps):
            hp.cycle(S)
            pushes_local += S * hp.n_particles
            if k + 1 < args.steps:
                m = torch.cuda.Event(enable_timing=True)
                m.record(stream)
                marks.append(m)
        e1.record(stream)
        marks.append(e1)
        torch.cuda.synchronize()
        barrier()
    launches = vpic.vpic_kernel_launches() - launches0
    hp.record_advance = False
    ms = e0.elapsed_time(e1)
    step_ms = [a.elapsed_time(b) for a, b in zip(marks[:-1], marks[1:])]
    adv = [(a.elapsed_time(b), n) for a, b, n in hp.adv_events]
    adv_ms = sum(t for t, _ in adv) / len(adv)
    nsp = len(hp.species)
    by_step = [round(sum(adv[(c * S + k) * nsp + j][0] for c in range(args.steps) for j in range(nsp))
                     / (args.steps * nsp), 3) for k in range(S)]
    by_species = {sp.name: [round(sum(adv[(c * S + k) * nsp + j][0] for c in range(args.steps))
                                  / args.steps, 3) for k in range(S)]
                  for j, sp in enumerate(hp.species)}
    sort_ms = {}
    for a, b, name in hp.sort_events:
        sort_ms.setdefault(name, []).append(a.elapsed_time(b))
    sort_ms = {k: round(sum(v) / len(v), 3) for k, v in sort_ms.items()}
    adv_np = sum(n for _, n in adv) / len(adv)
    t = torch.tensor([ms, float(pushes_local), float(n_local), float(hp.n_particles)],
                     dtype=torch.float64, device=red_dev)
    if world > 1:
        tmax = t.clone()
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        tsum = t.clone()
        dist.all_reduce(tsum, op=dist.ReduceOp.SUM)
        ms_max, pushes, ntot, nend = float(tmax[0]), float(tsum[1]), float(tsum[2]), float(tsum[3])
    else:
        ms_max, pushes, ntot, nend = ms, float(pushes_local), float(n_local), float(hp.n_particles)
    # global particle count: conserved by every exchange (no absorbing walls here)
    conservation = {"particles_start": int(ntot), "particles_end": int(nend), "ok": int(ntot) == int(nend)}
    value = pushes / (ms_max / 1e3)

    # ---- e2e: host (pinned) -> device inputs and device -> host results inside the timed region.
    # e2e: every step uploads the particles + fields and reads back the step's
    # result, jf (the current density the push produces for the field solver);
    # e2e_state_roundtrip additionally reads every particle back each step.
    e2e = e2e_rt = None
    if not args.no_e2e and not args.profile:
        host_in = [torch.from_numpy(np.ascontiguousarray(p).view(np.float32).reshape(-1, 8)).pin_memory()
                   for p in parts]
        f_host = torch.from_numpy(fields).pin_memory()
        jf_host = torch.empty(tuple(hp.jf.shape), dtype=torch.float32, pin_memory=True)
        h2d = sum(h.numel() * 4 for h in host_in) + f_host.numel() * 4

        def timed_e2e(outs):
            torch.cuda.synchronize()
            barrier()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            n = hp.run_host_cycles(host_in, outs, f_host, jf_host, args.steps, S)
            a1.record(stream)
            torch.cuda.synchronize()
            barrier()
            t = torch.tensor([a0.elapsed_time(a1), float(n)], dtype=torch.float64, device=red_dev)
            if world > 1:
                tm = t.clone(); dist.all_reduce(tm, op=dist.ReduceOp.MAX)
                ts = t.clone(); dist.all_reduce(ts, op=dist.ReduceOp.SUM)
                t = torch.stack([tm[0], ts[1]])
            return float(t[1]) / (float(t[0]) / 1e3)

        e2e = {"value": timed_e2e(None), "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": jf_host.numel() * 4,
               "result": "jf (current density) read back every step",
               "api": "vpic_run_host (C ABI): particles + fields uploaded from pinned host memory and jf "
                      "downloaded every step (one step = one sort period), copies pipelined on the "
                      "library's copy streams"}
        if world == 1:   # (N > 1: 17 GB more pinned host memory per rank; skipped)
            host_out = [torch.empty(tuple(h.shape), dtype=torch.float32, pin_memory=True)
                        for h in host_in]
            e2e_rt = {"value": timed_e2e(host_out), "unit": UNIT, "h2d_bytes_per_step": h2d,
                      "d2h_bytes_per_step": sum(h.numel() * 4 for h in host_out) + jf_host.numel() * 4,
                      "result": "every particle and jf read back every step"}

    if rank != 0:
        return
    # ---- roofline of the dominant kernel (k_advance: one launch = one species)
    peak, peak_kind = hbm_peak()
    ncell = g.nx * g.ny * g.nz
    alg_bytes = 64.0 * adv_np + (80.0 + 48.0) * ncell
    achieved = alg_bytes / (adv_ms / 1e3) / 1e9
    traffic, tinfo = committed_traffic("k_advance", wl.name)
    adv_share = sum(t for t, _ in adv) / ms
    clocks = clk.summary()
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
        "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic (seeded Philox; " + {
            "uniform": "uniform thermal e/ion plasma, quiet start",
            "harris": "Harris sheet: sech^2 density + background, tanh cB_x, drifting species, "
                      "reflecting z",
            "lpi": "laser-plasma slab: hot drifting electrons, cold ions, static laser ey = cbz"}[wl.kind] + ")",
        "config": {"workload": wl.name, "cells_per_gpu": [g.nx, g.ny, g.nz],
                   "global_cells": ([g.gnx or g.nx, g.ny * inputs.process_grid(world)[1],
                                     g.nz * inputs.process_grid(world)[2]] if strong else None),
                   "ppc_per_species": wl.ppc,
                   "species": len(wl.species), "particles": int(ntot), "sort_every": S,
                   "order": args.order, "shuffled": bool(args.shuffle), "math": args.math,
                   "deposit": args.deposit if args.deposit != "auto" else
                   "auto (warp; smem per species while its thermal spread since the sort is 0.4-1.3 cells)",
                   "kernel": args.kernel,
                   "parallelism": ("loopback1" if args.loopback and world == 1 else
                                   f"block 0 of {args.block_of} (1 GPU, no exchange)" if world == 1 and args.block_of > 1
                                   else f"domain{world}"),
                   "box_cells": [box.nx, box.ny, box.nz],
                   "field_solve": bool(args.field_solve),
                   "exchange": ("nccl" if (args.exchange == "nccl" or not hp.device_exchange) else "device")
                               if (world > 1 or args.loopback) else "none",
                   "migration": ("rounds" if args.migration == "rounds" else "single")
                                if (world > 1 or args.loopback) else "none",
                   "cpu_bind": cpu_bind,
                   "l2": f"no flush: inputs ({32 * n_local / 1e9:.1f} GB of particles per GPU) >> 126 MB L2"},
        "per_gpu": value / world,
        "step_ms_rank0": {"median": round(statistics.median(step_ms), 3), "min": round(min(step_ms), 3),
                          "max": round(max(step_ms), 3)},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "peak_kind": peak_kind,
                     "kernel": "k_advance (advance_p, one species per launch)",
                     "alg_bytes_per_launch": alg_bytes, "avg_launch_ms": adv_ms,
                     "share_of_step": adv_share, "frac_of_8TBs": achieved / 8000.0,
                     "avg_launch_ms_by_step_since_sort": by_step,
                     "launch_ms_by_species_step": by_species},
        "sort_ms_by_species": sort_ms,
        "comm": comm,
        "conservation": conservation,
        "clocks": clocks,
        "gpu_launches": launches,
        "e2e": e2e,
        "e2e_state_roundtrip": e2e_rt,
    }
    if not args.no_cpu_baseline and not args.profile and world == 1:
        out["cpu_baseline"] = cpu_baseline(args)
    print(json.dumps(out), flush=True)


def replace_grid(g, **kw):
    from dataclasses import replace
    return replace(g, **kw)


def spawn_ranks(n: int) -> int:
    """`bench.py --gpus N` without a torchrun environment: launch N ranks
    (one per GPU, NCCL) through torch.distributed.run on 127.0.0.1 and
    return their exit code; rank 0 prints the JSON line."""
    import socket
    import torch
    have = torch.cuda.device_count()
    if have < n and not SHARE_GPU:
        print(f"bench.py: --gpus {n} but {have} GPU(s) visible", file=sys.stderr, flush=True)
        return 2
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    print(f"bench.py: launching {n} ranks: {' '.join(cmd)}", file=sys.stderr, flush=True)
    return subprocess.call(cmd)


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if args.impl == "reference":
        reference_arm(args, rank, world)
        return
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(args.gpus))
    if world > 1:
        import torch
        import torch.distributed as dist
        if SHARE_GPU:
            os.environ["NCCL_HOSTID"] = f"vpic-bench-{rank}"
            os.environ.setdefault("NCCL_SOCKET_IFNAME", "lo")
            os.environ.setdefault("NCCL_IB_DISABLE", "1")
        torch.cuda.set_device(0 if SHARE_GPU else int(os.environ.get("LOCAL_RANK", "0")))
        dist.init_process_group("gloo" if SHARE_GPU else "nccl")
        if rank == 0:
            print(f"bench.py: NCCL process group initialised, nranks={dist.get_world_size()}",
                  file=sys.stderr, flush=True)
    try:
        our_arm(args, rank, world)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()

"""The multi-GPU exchange (csrc/migrate.cu) with several real ranks, against
the oracle's single-domain run ("non-blocking point-to-point
with up to six neighbors"; "exchanging particles").

tests/multirank_worker.py (one process per rank, torch.distributed.run)
splits a 16x8x8 box with reflecting z walls over the ranks (process grids
2x1x1, 2x2x1, 2x2x2), runs 3 IEEE-math PIC steps in each exchange mode and
gathers the particles on global voxel indices: they must equal the oracle's
bit for bit (as a multiset) and jf must be within T1 of the oracle's on every
edge.
* on the build's 1-GPU boxes: 2, 4 and 8 ranks sharing GPU 0, the NCCL modes
  (face rounds, single 26-neighbour round) over NCCL's socket transport;
* on a multi-GPU box (skipped otherwise): one rank per GPU, every mode incl.
  the device-initiated (NVLink symmetric-memory) ones.
"""
import os
import subprocess
import sys

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def _ngpu():
    return torch.cuda.device_count() if torch.cuda.is_available() else 0


def _free_gpu_memory():
    """The subprocesses need the GPU memory this pytest process may still
    cache from earlier (full-size) tests."""
    import gc
    gc.collect()
    if torch.cuda.is_available():
        torch.cuda.synchronize()
        torch.cuda.empty_cache()


def _run_and_compare(orc, tmp_path, nranks, env_extra, modes):
    _free_gpu_memory()
    import multirank_worker as W
    from paper_conf_sc_tanlta25_b200 import _build
    from paper_conf_sc_tanlta25_b200 import inputs
    from test_gpu_fields import assert_jf_t1, oracle_steps
    _build.build()
    out = str(tmp_path / "res.npz")
    port = 29500 + (os.getpid() % 1000) + nranks
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nranks}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(HERE, "multirank_worker.py"),
           out]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=800, env={**os.environ, **env_extra})
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    res = np.load(out)
    wl = W.global_workload()
    g = wl.grid
    parts = inputs.make_species_particles(wl)
    po, jo, jabs, _ = oracle_steps(orc, g, wl, parts, inputs.make_fields(g, 0.05), wl.steps)
    key = lambda a: np.sort(np.ascontiguousarray(a).view(np.dtype((np.void, 32))))
    for exch, mig in modes:
        for k in range(len(parts)):
            got = res[f"{exch}_{mig}_p{k}"]
            assert got.size == po[k].size, (exch, mig, k, got.size, po[k].size)
            assert np.array_equal(key(got), key(po[k])), (exch, mig, k)
        assert_jf_t1(g, res[f"{exch}_{mig}_jf"], jo, jabs)


@pytest.mark.timeout(600)
@pytest.mark.parametrize("nranks", [2, 4, 8])
def test_multirank_nccl_exchange_one_gpu_matches_oracle(orc, tmp_path, nranks):
    """The same worker with every rank on GPU 0 (MR_ONE_GPU): NCCL refuses two
    ranks of a communicator on one device of one host, so each rank poses as
    its own host (NCCL_HOSTID) and the ranks exchange through NCCL's socket
    transport on the loopback interface.  This runs migrate.cu's real
    multi-rank NCCL code -- several distinct peers, 2x1x1 / 2x2x1 / 2x2x2
    process grids, face rounds and the single 26-neighbour round -- on the
    build's 1-GPU boxes (the device-initiated modes need NVLink peers)."""
    sys.path.insert(0, HERE)
    import multirank_worker as W
    _run_and_compare(orc, tmp_path, nranks, {"MR_ONE_GPU": "1"}, [m for m in W.MODES if m[0] == "nccl"])


@pytest.mark.timeout(900)
def test_multirank_exchange_matches_oracle(orc, tmp_path):
    """On as many GPUs as the box has (8, 4 or 2: process grids 2x2x2,
    2x2x1, 2x1x1)."""
    nranks = max([n for n in (2, 4, 8) if n <= _ngpu()], default=0)
    if nranks == 0:
        pytest.skip(f"needs >= 2 GPUs, {_ngpu()} visible")
    sys.path.insert(0, HERE)
    import multirank_worker as W
    _run_and_compare(orc, tmp_path, nranks, {}, W.MODES)


@pytest.mark.timeout(900)
def test_bench_multirank_path_on_one_gpu():
    """bench.py's N > 1 path end to end (self-launch of the ranks, process
    grid, NCCL communicator, migration, max-over-ranks timing, the global
    conservation check, the C-ABI e2e leg) with 2 ranks sharing GPU 0
    (VPIC_BENCH_SHARE_GPU: gloo for torch.distributed, the library's NCCL
    over sockets; a functional test, not a measurement), on the f3 strong-
    scaling box."""
    import json
    _free_gpu_memory()
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env["VPIC_BENCH_SHARE_GPU"] = "1"
    r = subprocess.run([sys.executable, os.path.join(os.path.dirname(HERE), "bench.py"), "--gpus", "2",
                        "--config", "5", "--steps", "1", "--warmup", "1", "--no-cpu-baseline",
                        "--exchange", "nccl"], capture_output=True, text=True, env=env, timeout=800)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-3000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["n_gpus"] == 2 and line["scaling"] == "strong"
    assert line["comm"]["nranks"] == 2 and line["comm"]["vpic_ctx_nranks"] == 2
    assert line["conservation"]["ok"]
    assert line["e2e"]["value"] > 0

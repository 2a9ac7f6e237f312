"""The multi-GPU exchange (csrc/migrate.cu) across real GPUs, against the
oracle's single-domain run ("non-blocking point-to-point
with up to six neighbors"; "exchanging particles").

Skipped unless >= 2 GPUs are visible (the build's own boxes have one; the
one-GPU loopback tests in test_gpu_fields.py run the same code with a self
peer).  tests/multirank_worker.py runs each exchange mode -- NCCL rounds,
NCCL single-round, device-initiated rounds, device-initiated single-round --
for 3 IEEE-math PIC steps of a 16x8x8 box (walls on z) split over the ranks;
the particles (as a multiset, on global voxel indices) must equal the
oracle's bit for bit and jf must be within T1 of the oracle's on every edge.
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


@pytest.mark.timeout(900)
def test_multirank_exchange_matches_oracle(orc, tmp_path):
    """On as many GPUs as the box has (8, 4 or 2: process grids 2x2x2,
    2x2x1, 2x1x1)."""
    nranks = max([n for n in (2, 4, 8) if n <= _ngpu()], default=0)
    if nranks == 0:
        pytest.skip(f"needs >= 2 GPUs, {_ngpu()} visible")
    sys.path.insert(0, HERE)
    import multirank_worker as W
    from paper_conf_sc_tanlta25_b200 import _build
    from paper_conf_sc_tanlta25_b200 import inputs
    from test_gpu_fields import assert_jf_t1, oracle_steps
    _build.build()
    out = str(tmp_path / "res.npz")
    port = 29500 + (os.getpid() % 1000)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nranks}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(HERE, "multirank_worker.py"),
           out]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=800)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    res = np.load(out)
    wl = W.global_workload()
    g = wl.grid
    parts = inputs.make_species_particles(wl)
    po, jo, jabs, _ = oracle_steps(orc, g, wl, parts, inputs.make_fields(g, 0.05), wl.steps)
    key = lambda a: np.sort(np.ascontiguousarray(a).view(np.dtype((np.void, 32))))
    for exch, mig in W.MODES:
        for k in range(len(parts)):
            got = res[f"{exch}_{mig}_p{k}"]
            assert got.size == po[k].size, (exch, mig, k, got.size, po[k].size)
            assert np.array_equal(key(got), key(po[k])), (exch, mig, k)
        assert_jf_t1(g, res[f"{exch}_{mig}_jf"], jo, jabs)

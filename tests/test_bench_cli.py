"""bench.py's launch contract on a host without enough GPUs: `--gpus N`
without a torchrun environment launches N ranks itself (torch.distributed.run
on 127.0.0.1) -- here, with fewer GPUs visible than asked for, it must refuse
loudly (exit 2, a one-line reason) rather than run one process and report
n_gpus 1."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_gpus_n_without_enough_gpus_refuses():
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env["CUDA_VISIBLE_DEVICES"] = ""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1",
                        "--warmup", "3"], capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode == 2, (r.returncode, r.stdout[-500:], r.stderr[-500:])
    assert "--gpus 2 but 0 GPU(s) visible" in r.stderr

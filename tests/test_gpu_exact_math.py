"""csrc/exact_math.cuh (the branch-free correctly rounded sqrt / reciprocal of
the push's half displacement) against the CUDA library's __fsqrt_rn /
__frcp_rn: every float in [1, 2^26) and 2^28 random larger ones."""
import os
import subprocess

import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def test_exact_math_bitexact(tmp_path):
    exe = str(tmp_path / "exact_math_check")
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                           os.path.join(HERE, "exact_math_check.cu"), "-o", exe])
    r = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "mismatches 0," in r.stdout

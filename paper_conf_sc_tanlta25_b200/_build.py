"""Build libvpic.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

    python -m paper_conf_sc_tanlta25_b200._build [--force] [--verbose]

advance_p.cu is compiled twice: IEEE (-fmad=false, correctly rounded div/sqrt;
bit-exact with the oracle) and FAST (FMA + approximate rsqrt/division).
cudart is linked statically; NCCL is the libnccl.so.2 shipped with torch
(nvidia-nccl wheel), found through an rpath.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
BUILD = os.path.join(HERE, "build")
LIB = os.path.join(HERE, "libvpic.so")
ROOT = os.path.dirname(HERE)

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
          "--expt-relaxed-constexpr"]


def nccl_dirs():
    import importlib.util
    spec = importlib.util.find_spec("nvidia.nccl")
    if spec is None or not spec.submodule_search_locations:
        raise RuntimeError("nvidia-nccl (torch's NCCL) not found; cannot build libvpic.so")
    base = list(spec.submodule_search_locations)[0]
    return os.path.join(base, "include"), os.path.join(base, "lib")


def _units():
    inc, _ = nccl_dirs()
    I = ["-I", inc, "-I", os.path.join(ROOT, "include")]
    return [
        ("advance_fast.o", "advance_p.cu", ["-DVPIC_IEEE=0", "-fmad=true"]),
        ("advance_ieee.o", "advance_p.cu", ["-DVPIC_IEEE=1", "-fmad=false", "-prec-div=true",
                                            "-prec-sqrt=true"]),
        ("grid_ops.o", "grid_ops.cu", ["-fmad=false"]),
        ("sort.o", "sort.cu", []),
        ("migrate.o", "migrate.cu", []),
        ("gather_scatter.o", "gather_scatter.cu", []),
        ("diagnostics.o", "diagnostics.cu", ["-fmad=false"]),
        ("abi.o", "abi.cu", []),
        ("host_driver.o", "host_driver.cu", []),
    ], I


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    units, I = _units()
    headers = glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(ROOT, "include", "vpic.h"),
                                                       os.path.abspath(__file__)]
    objs = []
    jobs = []
    for obj, src, extra in units:
        o = os.path.join(BUILD, obj)
        s = os.path.join(CSRC, src)
        objs.append(o)
        if force or _stale(o, [s] + headers):
            jobs.append(["nvcc", *ARCH, *COMMON, *extra, *I, "-c", s, "-o", o])

    def run(cmd):
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("nvcc failed:\n" + " ".join(cmd) + "\n" + r.stdout + r.stderr)
        return cmd[-3], r.stdout + r.stderr

    with ThreadPoolExecutor(max(1, min(len(jobs), os.cpu_count() or 1))) as ex:
        for src, log in ex.map(run, jobs):
            if verbose:
                print(f"== {src}\n{log}")
    if force or jobs or _stale(LIB, objs):
        _, libdir = nccl_dirs()
        cmd = ["nvcc", *ARCH, "-shared", "-cudart", "static", "-o", LIB + ".tmp", *objs,
               "-L", libdir, "-l:libnccl.so.2", "-Xlinker", f"-rpath,{libdir}"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("link failed:\n" + " ".join(cmd) + "\n" + r.stdout + r.stderr)
        os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="--verbose" in sys.argv))

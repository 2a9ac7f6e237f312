"""Mutation test of the GPU parity tests (dev tool).

Each mutation plants a plausible bug in the CUDA path (a sign, an index, a
dropped term, a lost partial sum, an unstable rank...).  `build` compiles one
library per mutation next to the product one (libvpic_mut<k>.so; only the
mutated translation units are recompiled); `run` (on a GPU box) runs the
parity tests against each through VPIC_LIB and reports whether they reject
it.  A surviving mutation is a bug the parity tests would not see.

    python tools/kernel_mutations.py build
    python tools/kernel_mutations.py run [--out profiles/r02/kernel_mutations.txt]
"""
import argparse
import os
import shutil
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sc_tanlta25_b200")
sys.path.insert(0, ROOT)

# (name, file, old, new): `old` must occur exactly once in the file
MUTATIONS = [
    # ---- push (advance_p.cu)
    ("Boris tan correction truncated after v2/3", "advance_p.cu",
     "float v3 = v0 * (ONE + v2 * (ONE_THIRD + v2 * TWO_FIFTEENTHS));", "float v3 = v0 * (ONE + v2 * ONE_THIRD);"),
    ("half displacement: cdt_dx / cdt_dy swapped", "advance_p.cu",
     "  ux = MUL_RN(ux, cdt_dx);\n  uy = MUL_RN(uy, cdt_dy);", "  ux = MUL_RN(ux, cdt_dy);\n  uy = MUL_RN(uy, cdt_dx);"),
    ("exact reciprocal without its correction step", "exact_math.cuh",
     'asm("fma.rn.f32 %0, %1, %2, %1;" : "=f"(o) : "f"(r), "f"(t));', "o = r; (void)t;"),
    # ---- move_p / deposit
    ("periodic/local neighbour keeps the offset sign", "advance_p.cu",
     "  p.i = boundary ? v - dir * (n - 1) * stride : v + dir * stride;\n  if (axis == 0) p.dx = -d;",
     "  p.i = boundary ? v - dir * (n - 1) * stride : v + dir * stride;\n  if (axis == 0) p.dx = d;"),
    ("move_p drops the last streak's deposit", "advance_p.cu",
     "    deposit_lane(acc, p.i, c);\n    apply_streak(p, rx, ry, rz, st);\n    if (st.axis == 3) return ghost;",
     "    if (st.axis != 3) deposit_lane(acc, p.i, c);\n    apply_streak(p, rx, ry, rz, st);\n    if (st.axis == 3) return ghost;"),
    ("ACCUMULATE_J: v0 sign", "advance_p.cu", "  v0 = SUB_RN(v4, v1);", "  v0 = SUB_RN(v1, v4);"),
    ("warp butterfly subtracts", "advance_p.cu", "      v[k] = keep + __shfl_xor_sync(FULL, send, bit);",
     "      v[k] = keep - __shfl_xor_sync(FULL, send, bit);"),
    ("warp deposit: segment sum to the neighbouring slot", "advance_p.cu",
     "      if (!(lane & 1) && lane < 24) red_add(acc + 12 * (int64_t)seg + (lane >> 1), s);",
     "      if (!(lane & 1) && lane < 24) red_add(acc + 12 * (int64_t)seg + ((lane >> 1) ^ 1), s);"),
    ("smem deposit carry overwritten instead of accumulated", "advance_p.cu",
     "        for (int j = 0; j < 12; ++j) cr->v[j] += cm[j];", "        for (int j = 0; j < 12; ++j) cr->v[j] = cm[j];"),
    ("smem deposit: segment sum to the neighbouring slot", "advance_p.cu",
     "      if (!(lane & 1) && lane < 24) red_add(acc + 12 * (int64_t)seg + (lane >> 1), sum);\n    }\n    doneA",
     "      if (!(lane & 1) && lane < 24) red_add(acc + 12 * (int64_t)seg + ((lane >> 1) ^ 1), sum);\n    }\n    doneA"),
    ("carry-first: stragglers of set A not deposited", "advance_p.cu",
     "        if (sA) deposit_lane(acc, keyA, cA);", "        (void)sA;"),
    ("carry-first: A items of the carried voxel dropped", "advance_p.cu",
     "        if (inCA) t += cA[j];", "        (void)inCA;"),
    ("carry-first: B items of the chunk's last voxel not carried", "advance_p.cu",
     "          if (inLB) t += cB[j];", "          (void)inLB;"),
    ("carry-first: new carry keeps the old voxel", "advance_p.cu",
     "        cr->key = last;", "        cr->key = ck >= 0 ? ck : last;"),
    ("chunk runs: the next run starts one chunk late", "advance_p.cu",
     "c + RUN * GW - (RUN - 1)", "c + RUN * GW - (RUN - 2)"),
    ("TMA kernel: B crossers queued over A's slots", "advance_p.cu",
     "wrapn<QCAP>(qhead + qn + __popc(cmA) + __popc(cmB & lt))", "wrapn<QCAP>(qhead + qn + __popc(cmB & lt))"),
    ("TMA kernel: B keys written to A's slots", "advance_p.cu",
     "if (B.valid && B.inbnds) g.keys_out[first + 32 + lane]", "if (B.valid && B.inbnds) g.keys_out[first + lane]"),
    # ---- interpolator / unload (grid_ops.cu)
    ("interpolator: ex d2exdydz sign", "grid_ops.cu",
     "      w0 = e000.x; w1 = e010.x; w2 = e001.x; w3 = e011.x;\n      o0.x = fourth * ((w3 + w0) + (w1 + w2));\n"
     "      o0.y = fourth * ((w3 - w0) + (w1 - w2));\n      o0.z = fourth * ((w3 - w0) - (w1 - w2));\n"
     "      o0.w = fourth * ((w3 + w0) - (w1 + w2));",
     "      w0 = e000.x; w1 = e010.x; w2 = e001.x; w3 = e011.x;\n      o0.x = fourth * ((w3 + w0) + (w1 + w2));\n"
     "      o0.y = fourth * ((w3 - w0) + (w1 - w2));\n      o0.z = fourth * ((w3 - w0) - (w1 - w2));\n"
     "      o0.w = fourth * ((w3 + w0) + (w1 - w2));"),
    ("interpolator: dcbxdx sign", "grid_ops.cu", "o3.y = half * (b100.x - b000.x);", "o3.y = half * (b000.x - b100.x);"),
    ("unload jx: z neighbour for the -y quadrant", "grid_ops.cu", "__ldg(a + 3 * vy).y", "__ldg(a + 3 * vz).y"),
    ("advance_b: curl term sign", "grid_ops.cu", "b.x -= py * (ey1.z - e.z) - pz * (ez1.y - e.y);",
     "b.x -= py * (ey1.z - e.z) + pz * (ez1.y - e.y);"),
    ("advance_e: current enters with + sign", "grid_ops.cu", "- cj * j.y;", "+ cj * j.y;"),
    # ---- migrate / rho
    ("arrival movers index from 0 instead of np", "migrate.cu",
     "m.dispx = d.x; m.dispy = d.y; m.dispz = d.z; m.idx = (int32_t)(np + k);",
     "m.dispx = d.x; m.dispy = d.y; m.dispz = d.z; m.idx = (int32_t)k;"),
    ("hole backfill copies the wrong way", "migrate.cu",
     "  const int64_t n = (int64_t)*nlow;\n  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n;\n"
     "       k += (int64_t)gridDim.x * blockDim.x)\n    p[low[k]] = p[surv[k]];",
     "  const int64_t n = (int64_t)*nlow;\n  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n;\n"
     "       k += (int64_t)gridDim.x * blockDim.x)\n    p[surv[k]] = p[low[k]];"),
    ("rho: (1-dx) / (1+dx) weights swapped", "diagnostics.cu",
     "const float wx[2] = {1.0f - a.x, 1.0f + a.x};", "const float wx[2] = {1.0f + a.x, 1.0f - a.x};"),
    # ---- sort (sort.cu)
    ("radix rank counts later lanes (unstable)", "sort.cu",
     "      const uint32_t r = cur + __popc(peers & lt);", "      const uint32_t r = cur + __popc(peers & ~lt & ~(1u << lane));"),
    ("gather (strided / tiled orders) swaps the record halves", "sort.cu",
     "\n        const float4 *a = src + 2 * (int64_t)sidx[j] + (t & 1);",
     "\n        const float4 *a = src + 2 * (int64_t)sidx[j] + ((t & 1) ^ 1);"),
    ("fused record pass (standard order) swaps the record halves", "sort.cu",
     "\n            const float4 *a = src + 2 * (int64_t)sidx[j] + (t & 1);",
     "\n            const float4 *a = src + 2 * (int64_t)sidx[j] + ((t & 1) ^ 1);"),
    ("fused record pass: permutation written one slot off", "sort.cu",
     "rec.perm64[dpos[j]] = sidx[j];", "rec.perm64[dpos[j] ^ 1] = sidx[j];"),
    ("tiled rank key: chunk from key - min_k (R4)", "sort.cu",
     "        ck = (KeyT)((uint64_t)(k / T - chunk0) * max_r + (uint64_t)r);",
     "        ck = (KeyT)((uint64_t)((k - min_k) / T) * max_r + (uint64_t)r);"),
]

UNITS = {"advance_p.cu": ["advance_fast.o", "advance_ieee.o"], "exact_math.cuh": ["advance_fast.o", "advance_ieee.o"],
         "sort.cu": ["sort.o"], "grid_ops.cu": ["grid_ops.o"], "migrate.cu": ["migrate.o"],
         "diagnostics.cu": ["diagnostics.o"]}

TESTS = ("ieee_bitexact or fast_tolerance or sort_parity or edge_cases or unload_parity or ghost_fill "
         "or keyed or sort_captures or chunk_edges or one_cta or runs_wrap or 64bit or absorb_movers "
         "or test_gpu_fields or test_gpu_diagnostics")


def build(only=None):
    from paper_conf_sc_tanlta25_b200 import _build
    _build.build()
    inc, libdir = _build.nccl_dirs()
    units, I = _build._units()
    unit_flags = {o: (src, extra) for o, src, extra in units}
    for k, (name, fname, old, new) in enumerate(MUTATIONS):
        if only is not None and k not in only:
            continue
        path = os.path.join(PKG, "csrc", fname)
        src = open(path).read()
        if src.count(old) != 1:
            print(f"SKIP {name}: pattern occurs {src.count(old)} times")
            continue
        with tempfile.TemporaryDirectory() as td:
            csrc = os.path.join(td, "pkg", "csrc")   # (csrc includes ../../include/vpic.h)
            shutil.copytree(os.path.join(PKG, "csrc"), csrc)
            os.symlink(os.path.join(ROOT, "include"), os.path.join(td, "include"))
            with open(os.path.join(csrc, fname), "w") as f:
                f.write(src.replace(old, new))
            objs = []
            for o, (s, extra) in unit_flags.items():
                if o in UNITS[fname]:
                    out = os.path.join(td, o)
                    cmd = ["nvcc", *_build.ARCH, *_build.COMMON, *extra, "-I", inc, "-I", os.path.join(ROOT, "include"),
                           "-c", os.path.join(csrc, s), "-o", out]
                    r = subprocess.run(cmd, capture_output=True, text=True)
                    if r.returncode != 0:
                        raise RuntimeError(f"mutant {k} ({name}) does not compile:\n{r.stderr[-2000:]}")
                    objs.append(out)
                else:
                    objs.append(os.path.join(_build.BUILD, o))
            lib = os.path.join(PKG, f"libvpic_mut{k}.so")
            subprocess.run(["nvcc", *_build.ARCH, "-shared", "-cudart", "static", "-o", lib, *objs, "-L", libdir,
                            "-l:libnccl.so.2", "-Xlinker", f"-rpath,{libdir}"], check=True, capture_output=True)
        print(f"built mut{k}: {name}", flush=True)


def run(out, only=None):
    lines = []
    killed = total = 0
    todo = [(-1, ("control: the product library", None, None, None))] + list(enumerate(MUTATIONS))
    for k, (name, fname, old, new) in todo:
        if only is not None and k >= 0 and k not in only:
            continue
        lib = os.path.join(PKG, "libvpic.so" if k < 0 else f"libvpic_mut{k}.so")
        if not os.path.exists(lib):
            continue
        env = dict(os.environ, VPIC_LIB=lib)
        t0 = time.time()
        try:
            r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider",
                                "tests/test_gpu_parity.py", "tests/test_gpu_fields.py", "tests/test_gpu_diagnostics.py",
                                "-k", TESTS], cwd=ROOT, env=env, capture_output=True,
                               text=True, timeout=900)
            rc = r.returncode
            failed = [l for l in r.stdout.splitlines() if l.startswith("FAILED")]
        except subprocess.TimeoutExpired:
            rc, failed = -1, ["timeout"]
        dt = f"[{time.time() - t0:.0f} s]"
        if k < 0:
            lines.append(f"{'PASS' if rc == 0 else 'FAIL'} {name} {dt}")
            if rc != 0:
                print(r.stdout[-3000:])
                break
        elif rc != 0:
            total += 1
            killed += 1
            lines.append(f"KILLED {name} {dt} <- {failed[0][7:100] if failed else 'error rc=%d' % rc}")
        else:
            total += 1
            lines.append(f"SURVIVED {name} {dt}")
        print(lines[-1], flush=True)
    summary = f"{killed} of {total} kernel mutations rejected by the GPU parity tests"
    print(summary)
    if out:
        with open(out, "w") as f:
            f.write(__doc__.strip().splitlines()[0] + "\n" + summary + "\n" + "\n".join(lines) + "\n")


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("cmd", choices=["build", "run"])
    ap.add_argument("--out", default=None)
    ap.add_argument("--only", type=int, nargs="*", default=None, help="mutation indices")
    a = ap.parse_args()
    build(a.only) if a.cmd == "build" else run(a.out, a.only)

"""Mutation test of the oracle's pins (dev tool).

Each mutation is a plausible mistake in oracle/vpic_oracle.cpp -- a dropped
term, a wrong sign, a swapped index or operand, a misread of the paper's
algorithms.  The mutated oracle is built to a temporary library and the CPU
pin tests (tests/test_oracle_*.py, -m "not gpu") are run against it through
ORACLE_LIB; a mutation is KILLED when some pin fails.  A surviving mutation
means the pins cannot tell that mistake from the paper's method.

    python tools/oracle_mutations.py [--out profiles/r02/oracle_mutations.txt]
"""
import argparse
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "vpic_oracle.cpp")

# (name, old, new): `old` must occur exactly once in the source
MUTATIONS = [
    # ---- sort (Alg. 1 / Alg. 2, readings R1-R5)
    ("strided stride max_k-min_k+1 instead of max_k+1 (R5)",
     "new_keys[i] = (key - min_k) + r * (max_k + 1);", "new_keys[i] = (key - min_k) + r * (max_k - min_k + 1);"),
    ("tiled chunk from key-min_k instead of the raw key (R4)",
     "const int64_t chunk = (int64_t)keys[i] / tile_sz;", "const int64_t chunk = ((int64_t)keys[i] - min_k) / tile_sz;"),
    ("tiled id modulo T (R3)",
     "new_keys[i] = chunk * chunk_sz + tile * tile_sz + id;", "new_keys[i] = chunk * chunk_sz + tile * tile_sz + id % tile_sz;"),
    ("rank counts one too many (Alg. 2 L12)",
     "const int64_t tile = key_counts[id]++;", "const int64_t tile = ++key_counts[id];"),
    ("unstable sort (R1)",
     "std::stable_sort(perm.begin(), perm.end(),", "std::sort(perm.begin(), perm.end(),"),
    # ---- interpolator
    ("ex: d2exdydz sign",
     "fi[3] = fourth * ((w3 + w0) - (w1 + w2));", "fi[3] = fourth * ((w3 + w0) + (w1 - w2));"),
    ("ey: y/z neighbours swapped",
     "w0 = F(x, y, z, 1); w1 = F(x, y, z + 1, 1); w2 = F(x + 1, y, z, 1); w3 = F(x + 1, y, z + 1, 1);",
     "w0 = F(x, y, z, 1); w1 = F(x + 1, y, z, 1); w2 = F(x, y, z + 1, 1); w3 = F(x + 1, y, z + 1, 1);"),
    ("cbx: difference sign", "fi[13] = half * (w1 - w0);", "fi[13] = half * (w0 - w1);"),
    # ---- push
    ("gather hay: dy instead of dz", "const float hay = qdt_2mc * ((f_ey + dz * f_deydz)", "const float hay = qdt_2mc * ((f_ey + dy * f_deydz)"),
    ("gather cbx: dy instead of dx", "const float cbx = f_cbx + dx * f_dcbxdx;", "const float cbx = f_cbx + dy * f_dcbxdx;"),
    ("tan correction dropped (plain Boris, R11)",
     "float v3 = v0 * (one + v2 * (one_third + v2 * two_fifteenths));", "float v3 = v0;"),
    ("tan correction truncated after v2/3 (R11)",
     "float v3 = v0 * (one + v2 * (one_third + v2 * two_fifteenths));", "float v3 = v0 * (one + v2 * one_third);"),
    ("Boris second rotation not doubled", "    v4 += v4;\n    v0 = ux", "    v0 = ux"),
    ("Boris rotation cross product sign", "v0 = ux + v3 * (uy * cbz - uz * cby);", "v0 = ux + v3 * (uz * cby - uy * cbz);"),
    ("second half E kick dropped", "    /* half E kick */\n    ux += hax;\n    uy += hay;\n    uz += haz;\n    p->ux = ux;",
     "    /* half E kick */\n    p->ux = ux;"),
    ("gamma from the old momentum", "float v0 = qdt_2mc / std::sqrt(one + (ux * ux + (uy * uy + uz * uz)));",
     "float v0 = qdt_2mc / std::sqrt(one + ((float)p->ux * p->ux + ((float)p->uy * p->uy + (float)p->uz * p->uz)));"),
    ("half displacement: cdt_dx / cdt_dy swapped", "  ux *= cdt_dx;\n  uy *= cdt_dy;", "  ux *= cdt_dy;\n  uy *= cdt_dx;"),
    # ---- move_p (R12, R13)
    # (ties between faces, '<' vs '<=', only reorder zero-length streaks --
    #  their partials are exactly zero -- so that mutation is equivalent; the
    #  GPU edge-case parity tests check the kernels' tie handling bit for bit)
    ("end-of-track tie lost to a face inside move_p (R13)", "    float v3 = 2.0f;\n    int axis = 3;",
     "    float v3 = 2.0000002f;\n    int axis = 3;"),
    ("streak fraction not halved", "    v3 *= 0.5f;\n    /* streak half-displacement", "    /* streak half-displacement"),
    ("reflect keeps the momentum (R12)", "      (&p->ux)[axis] = -(&p->ux)[axis];\n", ""),
    ("periodic neighbour keeps the offset sign", "  p->i = (int32_t)nb;\n    (&p->dx)[axis] = -d;", "  p->i = (int32_t)nb;\n    (&p->dx)[axis] = d;"),
    # ---- deposit (ACCUMULATE_J)
    ("ACCUMULATE_J: v0 sign", "  v0 = v4 - v1;", "  v0 = v1 - v4;"),
    ("ACCUMULATE_J: (1+dZ) / (1-dZ) swapped", "  v4 = one + dZ;", "  v4 = one - dZ;"),
    ("ACCUMULATE_J: correction term sign", "  v0 += v5;", "  v0 -= v5;"),
    ("ACCUMULATE_J: correction term dropped", "const float v5 = q * sx * sy * sz * one_third;", "const float v5 = 0.0f * q * sx * sy * sz;"),
    ("ACCUMULATE_J: y component's transverse axes swapped", "accumulate_j(q, sy, mz, mx, v5,", "accumulate_j(q, sy, mx, mz, v5,"),
    # ---- unload
    ("unload jx: -y neighbour quadrant index", "A(x, y - 1, z, 1)", "A(x, y - 1, z, 2)"),
    ("unload jz: wrong neighbour", "A(x - 1, y, z, 9)", "A(x, y - 1, z, 9)"),
    # ---- rho, absorbed, continuity, field solver
    ("rho: (1+d) / (1-d) swapped", "wgt *= hi ? (1.0 + d[a]) : (1.0 - d[a]);", "wgt *= hi ? (1.0 - d[a]) : (1.0 + d[a]);"),
    ("remove_absorbed: remote-face movers removed too", "if (g->pbc[face] == 2) idx.push_back(i);", "idx.push_back(i);"),
    ("continuity residual: drho sign", "double r = drho, m = std::fabs(drho);", "double r = -drho, m = std::fabs(drho);"),
    ("advance_e: curl sign", "F(x, y, z, 0) += py * (cbz - F(x, y - 1, z, 6)) - pz * (cby - F(x, y, z - 1, 5))",
     "F(x, y, z, 0) += py * (cbz - F(x, y - 1, z, 6)) + pz * (cby - F(x, y, z - 1, 5))"),
    ("advance_b: forward difference on the wrong side", "F(x, y, z, 4) -= py * (F(x, y + 1, z, 2) - ez)",
     "F(x, y, z, 4) -= py * (ez - F(x, y - 1, z, 2))"),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("-k", default=None, help="only mutations whose name contains this")
    a = ap.parse_args()
    src = open(SRC).read()
    lines = []
    killed = 0
    todo = [m for m in MUTATIONS if not a.k or a.k in m[0]]
    with tempfile.TemporaryDirectory() as td:
        for k, (name, old, new) in enumerate(todo):
            n = src.count(old)
            if n != 1:
                lines.append(f"SKIP  {name}: pattern occurs {n} times")
                continue
            mut = os.path.join(td, f"m{k}.cpp")
            with open(mut, "w") as f:
                f.write(src.replace(old, new))
            lib = os.path.join(td, f"m{k}.so")
            subprocess.check_call(["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                                   "-fPIC", "-shared", "-I", os.path.join(ROOT, "oracle"), mut, "-o", lib])
            env = dict(os.environ, ORACLE_LIB=lib)
            try:
                r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "not gpu", "-p", "no:cacheprovider",
                                    "--timeout", "60",
                                    "tests/test_oracle_sort.py", "tests/test_oracle_interp_unload.py",
                                    "tests/test_oracle_push.py", "tests/test_oracle_rho.py", "tests/test_oracle_fields.py",
                                    "tests/test_oracle_gather_scatter.py"],
                                   cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
            except subprocess.TimeoutExpired:
                killed += 1
                lines.append(f"KILLED {name}  <- the pins time out (the mutated oracle does not terminate)")
                print(lines[-1], flush=True)
                continue
            if r.returncode != 0:
                killed += 1
                failed = [l for l in r.stdout.splitlines() if l.startswith("FAILED")]
                lines.append(f"KILLED {name}  <- {failed[0][7:80] if failed else 'error'}")
            else:
                lines.append(f"SURVIVED {name}")
            print(lines[-1], flush=True)
    summary = f"{killed} of {len(todo)} mutations killed by the CPU pins"
    print(summary)
    if a.out:
        with open(a.out, "w") as f:
            f.write(__doc__.strip().splitlines()[0] + "\n" + summary + "\n" + "\n".join(lines) + "\n")


if __name__ == "__main__":
    main()

"""Top CUDA source lines of an ncu report by instructions executed (dev tool).
    python tools/ncu_ex_lines.py rep.ncu-rep [N]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
hdr = rows[hdr_i]
ex = hdr.index("Instructions Executed")
def num(x):
    try:
        return int(x)
    except ValueError:
        return 0
agg = {}
for r in rows[hdr_i + 1:]:
    if len(r) != len(hdr) or not r[0].strip():
        continue
    k = (r[0], r[1].strip()[:90])
    agg[k] = agg.get(k, 0) + num(r[ex])
tot = sum(agg.values())
print("total warp instructions", tot)
for (ln, src), v in sorted(agg.items(), key=lambda x: -x[1])[:N]:
    print(f"{ln:>5} {v / 1e6:8.1f}M {100 * v / tot:5.1f}%  {src}")

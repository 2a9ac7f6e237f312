"""Top CUDA source lines of an ncu report by warp-stall samples (dev tool).
    python tools/ncu_lines.py rep.ncu-rep [N]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
extra = sys.argv[3:]   # e.g. -k regex:k_radix --launch-skip 0 -c 1
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"] + extra,
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
hdr = rows[hdr_i]
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_")]
def num(x):
    try:
        return int(x)
    except ValueError:
        return 0
data = [[c if j < 4 else num(c) for j, c in enumerate(r)] for r in rows[hdr_i + 1:] if len(r) == len(hdr)]
tot = sum(r[4] for r in data)
print("total samples", tot, " instr", sum(r[7] for r in data))
data.sort(key=lambda r: -r[4])
for r in data[:N]:
    s = r[4]
    st = sorted(((r[i], hdr[i][6:]) for i in stall_cols), reverse=True)[:3]
    print(f"{r[0]:>5} {100*s/tot:5.1f}% ex={r[7]/1e6:7.1f}M  {' '.join(f'{n}={v}' for v, n in st):60s} {r[1].strip()[:70]}")

"""Group an ncu report's SASS by execution count (dev tool)."""
import csv, io, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]; data = rows[2:]
ix = {h: i for i, h in enumerate(hdr)}
tot = sum(int(r[ix["Instructions Executed"]] or 0) for r in data)
print("total warp instr", tot)
groups = []
for r in data:
    ex = int(r[ix["Instructions Executed"]] or 0)
    smp = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    thr = r[ix["Avg. Threads Executed"]]
    bank = r[ix.get("L1 Conflicts Shared N-Way", 0)] if "L1 Conflicts Shared N-Way" in ix else ""
    if groups and groups[-1]["ex"] == ex:
        g = groups[-1]; g["n"] += 1; g["end"] = r[0][-5:]; g["smp"] += smp; g["ops"].append(r[1].split()[0] if r[1].split() else "")
    else:
        groups.append({"ex": ex, "n": 1, "start": r[0][-5:], "end": r[0][-5:], "smp": smp, "thr": thr, "ops": [r[1].split()[0] if r[1].split() else ""]})
thr_min = float(sys.argv[2]) if len(sys.argv) > 2 else 30e6
for g in groups:
    if g["ex"] * g["n"] > thr_min:
        ops = {}
        for o in g["ops"]:
            o = o.split(".")[0]
            ops[o] = ops.get(o, 0) + 1
        top = ",".join(f"{k}:{v}" for k, v in sorted(ops.items(), key=lambda x: -x[1])[:6])
        print(f'{g["start"]}-{g["end"]} n={g["n"]:4d} x {g["ex"]:>9} = {g["ex"]*g["n"]/1e6:7.0f}M thr={g["thr"]:>3} samples={g["smp"]:6d} {top}')

"""Aggregate an ncu --metrics gpu__time_duration.sum CSV launch list (dev tool)."""
import collections, csv, io, sys
lines = open(sys.argv[1]).read().splitlines()
start = [i for i, l in enumerate(lines) if l.startswith('"ID"')][0]
rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
agg = collections.OrderedDict()
for r in rows:
    name = r['Kernel Name'][:70]
    unit = r['Metric Unit']
    v = float(r['Metric Value'].replace(',', ''))
    v = v / 1e6 if unit in ('ns', 'nsecond') else v / 1e3 if unit in ('us', 'usecond') else v
    a = agg.setdefault(name, [0, 0.0]); a[0] += 1; a[1] += v
tot = sum(v[1] for v in agg.values())
for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{n:5d} {t:10.3f} ms {t / n:8.3f} ms/launch {100 * t / tot:5.1f}%  {k}")
print(f"total {tot:.3f} ms, {sum(v[0] for v in agg.values())} launches")

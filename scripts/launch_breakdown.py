"""Per-kernel time from an ncu gpu__time_duration launch list (CSV). Builder tooling."""
import csv, re, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hi]
ik, iv, iu = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
agg = collections.OrderedDict(); tot = 0
for r in rows[hi + 1:]:
    if len(r) <= iv:
        continue
    name = re.sub(r'\(.*', '', r[ik]).replace('void ', '')
    v = float(r[iv].replace(',', '')); u = r[iu]
    us = {'nsecond': v / 1e3, 'ns': v / 1e3, 'usecond': v, 'us': v, 'msecond': v * 1e3, 'ms': v * 1e3}[u]
    a = agg.setdefault(name, [0, 0.0]); a[0] += 1; a[1] += us; tot += us
for k, (c, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{us:9.1f} us {100 * us / tot:5.1f}% n={c:3d} {k}")
print(f"{tot:9.1f} us total")

"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) by kernel (builder tooling)."""
import csv, sys, collections, re
rows = list(csv.reader(open(sys.argv[1])))
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr_i]
ik, iv, iid = h.index("Kernel Name"), h.index("Metric Value"), h.index("ID")
agg = collections.OrderedDict()
seq = []
for r in rows[hdr_i + 1:]:
    if len(r) <= iv or not r[iv]:
        continue
    name = re.sub(r"\(.*", "", r[ik]).replace("void ", "")
    v = float(r[iv].replace(",", ""))
    unit = r[h.index("Metric Unit")]
    us = {"nsecond": v / 1e3, "ns": v / 1e3, "usecond": v, "us": v, "msecond": v * 1e3, "ms": v * 1e3, "second": v * 1e6, "s": v * 1e6}.get(unit, v)
    seq.append((int(r[iid]), name, us))
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += us
tot = sum(x[1] for x in agg.values())
for k, (c, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{us:10.1f} us {100 * us / tot:5.1f}%  n={c:4d}  {k}")
print(f"{tot:10.1f} us total ({len(seq)} launches)")
if len(sys.argv) > 2:
    for i, n, us in seq[: int(sys.argv[2])]:
        print(f"{i:5d} {us:9.1f} {n}")

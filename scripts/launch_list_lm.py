"""Summarise an ncu launch list (CSV, gpu__time_duration.sum) over liblmatch kernels only, plus the
last run launch by launch (builder tooling).  usage: launch_list_lm.py launches.csv "header line" """
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hi]
ik, iv, iid, iu = h.index("Kernel Name"), h.index("Metric Value"), h.index("ID"), h.index("Metric Unit")
seq = []
for r in rows[hi + 1:]:
    if len(r) <= iv or not r[iv]:
        continue
    name = re.sub(r"\(.*", "", r[ik]).replace("void ", "")
    if not name.startswith("lm::"):
        continue
    v = float(r[iv].replace(",", ""))
    us = {"nsecond": v / 1e3, "ns": v / 1e3, "usecond": v, "us": v, "msecond": v * 1e3, "ms": v * 1e3}.get(r[iu], v)
    seq.append((int(r[iid]), name, us))
last = max(i for i, (_, n, _) in enumerate(seq) if n == "lm::k_reset")
run = seq[last:]
agg = collections.OrderedDict()
for _, n, us in seq:
    a = agg.setdefault(n, [0, 0.0])
    a[0] += 1
    a[1] += us
tot = sum(a[1] for a in agg.values())
out = ["# " + sys.argv[2],
       "# gpu__time_duration.sum, --clock-control none; cold-cache serialised launches; liblmatch kernels only",
       "# (the synthetic generator's kernels run before create and are excluded)",
       "# totals over 5 runs (3 warm-up + 2 timed) + the one-time create kernels"]
for n, (c, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    out.append(f"{us:10.1f} us {100 * us / tot:5.1f}%  n={c:4d}  {n}")
out.append(f"{tot:10.1f} us total ({len(seq)} launches)")
rt = sum(us for _, _, us in run)
sw = sum(us for _, n, us in run if n.startswith("lm::k_sweep<") and n.endswith(", 0>"))
out.append("")
out.append(f"# the last (timed) run, launch by launch: {len(run)} launches, {rt:.1f} us serialised; "
           f"k_sweep share {100 * sw / rt:.1f}%")
for i, n, us in run:
    out.append(f"{i:6d} {us:9.1f} {n}")
print("\n".join(out))

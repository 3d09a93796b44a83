"""Group an ncu launch list (--metrics gpu__time_duration.sum,launch__grid_size[,dram__bytes_*]) by
(kernel, grid size): launches, mean us, total ms, DRAM MB per launch.

  python tools/launch_groups.py <launches.csv>
"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
ii, ki, mi, vi, ui = (h.index(c) for c in ("ID", "Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
sc = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1, "msecond": 1e3}
per = collections.OrderedDict()
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    d = per.setdefault(r[ii], {"name": r[ki].split("(")[0].replace("void ", "")[:48]})
    d[r[mi]] = float(r[vi].replace(",", "")) * sc.get(r[ui], 1)
g = collections.OrderedDict()
for d in per.values():
    key = (d["name"], int(d.get("launch__grid_size", 0)))
    a = g.setdefault(key, [0, 0.0, 0.0])
    a[0] += 1
    a[1] += d["gpu__time_duration.sum"]
    a[2] += d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
tot = sum(a[1] for a in g.values())
print(f"{'kernel':50s} {'grid':>6s} {'n':>5s} {'mean us':>9s} {'total ms':>9s} {'share':>6s} {'MB/launch':>9s}")
for (n, gs), (c, t, b) in sorted(g.items(), key=lambda kv: -kv[1][1]):
    print(f"{n:50s} {gs:6d} {c:5d} {t / c:9.1f} {t / 1e3:9.2f} {t / tot:6.3f} {b / c / 1e6:9.1f}")
print(f"total {tot / 1e3:.2f} ms")

#!/usr/bin/env python
"""Per-kernel totals (us per fit) of ncu launch lists: python tools/ncu_table.py a.csv b.csv ..."""
import collections
import csv
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    ki, mi, vi, idi = (hdr.index(k) for k in ("Kernel Name", "Metric Name", "Metric Value", "ID"))
    per = collections.OrderedDict()
    for r in rows[start + 1:]:
        per.setdefault(r[idi], {"name": r[ki]})[r[mi]] = float(r[vi].replace(",", "") or 0)
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0, 0.0])
    nfit = 0
    for v in per.values():
        n = v["name"].split("(")[0].replace("void ", "").replace("dtl::<unnamed>::", "")
        if "cub::" in v["name"] or "DeviceRadix" in v["name"]:
            n = "cub_sort"
        if n == "root_init_kernel":
            nfit += 1
        a = agg[n]
        a[0] += 1
        a[1] += v.get("gpu__time_duration.sum", 0) / 1e3
        a[2] += (v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0)) / 1e6
        a[3] += v.get("smsp__inst_executed.sum", 0) / 1e6
    nfit = max(nfit, 1)
    return {k: [x / nfit for x in a] for k, a in agg.items()}


tabs = [load(p) for p in sys.argv[1:]]
names = sorted(set().union(*tabs), key=lambda n: -tabs[0].get(n, [0, 0])[1])
print("kernel".ljust(34) + "".join(f"{'v%d us' % (i + 1):>10}{'MB':>8}{'Minst':>8}" for i in range(len(tabs))))
for n in names:
    line = n[:33].ljust(34)
    for t in tabs:
        a = t.get(n, [0, 0, 0, 0])
        line += f"{a[1]:10.1f}{a[2]:8.0f}{a[3]:8.1f}"
    print(line)
print("total".ljust(34) + "".join(f"{sum(a[1] for a in t.values()):10.1f}{'':16}" for t in tabs))

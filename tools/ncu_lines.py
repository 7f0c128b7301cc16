#!/usr/bin/env python
"""Instructions executed and stall samples per CUDA source line of one kernel in an ncu
report (measurement helper): python tools/ncu_lines.py REPORT KERNEL_REGEX [TOP]"""
import csv
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", "regex:" + kern,
                      "--launch-count", "1", "--print-source", "cuda,sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = None
fname = ""
agg = {}
cur = None
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        ie = hdr.index("Instructions Executed")
        st = hdr.index("Warp Stall Sampling (All Samples)")
        continue
    if hdr is None or len(r) <= ie:
        continue
    if r[0]:
        cur = (fname, int(r[0]), r[1][:90])
        continue
    if cur and r[ie].strip().isdigit():
        a = agg.setdefault(cur, [0, 0])
        a[0] += int(r[ie])
        a[1] += int(r[st] or 0)
tot = sum(v[0] for v in agg.values()) or 1
tst = sum(v[1] for v in agg.values()) or 1
print(f"total warp instructions {tot}, stall samples {tst}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{v[0] / tot:6.3f} {v[1] / tst:6.3f}  {k[0]}:{k[1]}  {k[2]}")

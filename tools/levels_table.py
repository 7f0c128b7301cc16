"""Per-level kernel durations (us) of the second fit in an ncu launch list (development aid)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/it_launches.csv")))
st = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
h = rows[st]; ki = h.index("Kernel Name"); vi = h.index("Metric Value")
seq = [(r[ki].split("(")[0].split("::")[-1].split("<")[0].replace("void ", ""), float(r[vi].replace(",", "")) / 1000)
       for r in rows[st + 1:]]
seq = seq[len(seq) // 2:]
lvl, cur = [], []
for n, v in seq:
    if n.startswith("select") and cur:
        lvl.append(cur); cur = []
    cur.append((n, v))
lvl.append(cur)
tot = 0.0
for i, l in enumerate(lvl):
    s = sum(v for n, v in l); tot += s
    print(i, f"{s:7.1f}", " ".join(f"{n[:10]}={v:.0f}" for n, v in l if not n.startswith("rs_")))
print(f"total {tot:.1f} us")

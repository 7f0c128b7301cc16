"""Per-launch times (us) of selected kernels in launch order, second half of an ncu launch list."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
pat = sys.argv[2].split(",") if len(sys.argv) > 2 else ["fused", "level_agg", "general"]
st = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
h = rows[st]; ki = h.index("Kernel Name"); vi = h.index("Metric Value")
seq = [(r[ki].split("(")[0].split("::")[-1], float(r[vi].replace(",", ""))) for r in rows[st + 1:]]
seq = seq[len(seq) // 2:]
line = []
for name, v in seq:
    if any(p in name for p in pat):
        line.append(f"{name[:14]}={v/1000:.0f}")
print(" ".join(line))

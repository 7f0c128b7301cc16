"""Per-CUDA-source-line instruction counts and stall samples from an ncu report
(`ncu -i rep --page source --csv --print-source cuda,sass`).  Usage: ncu_lines2.py rep [top] [kernel-regex]"""
import csv, subprocess, sys, collections
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
kf = ["-k", "regex:" + sys.argv[3]] if len(sys.argv) > 3 else []  # optional kernel-name filter
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"] + kf,
                     capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(out))
agg = collections.defaultdict(lambda: [0.0, 0.0, ""])
fname = "?"
hdr = None
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = {k: i for i, k in enumerate(r)}
        continue
    if hdr is None or len(r) < len(hdr):
        continue
    try:
        ln = int(r[0])
    except ValueError:
        continue
    def f(k):
        try:
            return float(r[hdr[k]].replace(",", ""))
        except Exception:
            return 0.0
    key = (fname, ln)
    agg[key][0] += f("Instructions Executed")
    agg[key][1] += f("Warp Stall Sampling (All Samples)")
    agg[key][2] = r[1][:100]
tot = sum(v[0] for v in agg.values())
tots = sum(v[1] for v in agg.values())
print(f"total instructions {tot:.3e}, stall samples {tots:.0f}")
for (fn, ln), (ins, st, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{fn}:{ln:5d} {ins/tot*100:5.1f}% ins {st/tots*100:5.1f}% stall | {src}")

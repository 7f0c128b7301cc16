"""Per-source-line totals of an ncu SASS source page (measurement helper, not part of the
library): aligns `ncu --page source --csv --print-source sass` rows with a local
`nvdisasm -g -c` listing of the same build (instruction order) and sums instructions
executed and stall samples per CUDA source line.
usage: python tools/sass_lines.py <ncu sass csv> <nvdisasm listing> <kernel substring> [top]"""
import csv, re, sys, collections

def ncu_rows(path):
    rows = list(csv.reader(open(path)))
    hdr = next(r for r in rows if r and r[0] == "Address")
    i = rows.index(hdr)
    out = []
    for r in rows[i + 1:]:
        if not r or r[0] == "Kernel Name":
            break
        out.append(dict(zip(hdr, r)))
    return out

def listing(path, kern):
    on = False
    cur = None
    res = []
    for ln in open(path).read().splitlines():
        if ln.startswith(".text.") and ln.rstrip().endswith(":"):
            on = kern in ln
            continue
        if not on:
            continue
        if ln.lstrip().startswith("//##"):
            m = re.search(r'line (\d+)', ln)
            fm = re.search(r'File "([^"]+)"', ln)
            if m:
                cur = (fm.group(1).split("/")[-1] if fm else "?", int(m.group(1)))
            continue
        m = re.match(r'\s*/\*([0-9a-f]{4,})\*/\s+(.*?);', ln)
        if m:
            res.append((cur, m.group(2).strip()))
    return res

rows = ncu_rows(sys.argv[1])
lst = listing(sys.argv[2], sys.argv[3])
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
print("ncu instrs", len(rows), "listing instrs", len(lst))
n = min(len(rows), len(lst))
op = lambda s: s.lstrip("@!P0123456789T ").split()[0].split(".")[0] if s.strip() else ""
mism = sum(1 for k in range(n) if op(rows[k]["Source"]) != op(lst[k][1]))
print("opcode mismatches", mism)
agg = collections.defaultdict(lambda: [0, 0])
tot_i = tot_s = 0
for k in range(n):
    ie = int(rows[k]["Instructions Executed"] or 0)
    ss = int(rows[k]["Warp Stall Sampling (All Samples)"] or 0)
    agg[lst[k][0]][0] += ie
    agg[lst[k][0]][1] += ss
    tot_i += ie; tot_s += ss
print("total warp instr", tot_i, "samples", tot_s)
for key, (ie, ss) in sorted(agg.items(), key=lambda t: -t[1][0])[:top]:
    print(f"{str(key):32s} instr {ie:10d} {100*ie/tot_i:5.1f}%  stall {100*ss/max(tot_s,1):5.1f}%")

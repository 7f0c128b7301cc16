#!/usr/bin/env python
"""Summarise an ncu launch list (CSV from `ncu --metrics gpu__time_duration.sum,
dram__bytes_read.sum,dram__bytes_write.sum ... --csv --log-file X`) of ONE bench step.

Writes <out>.md (per-kernel table: launches, device time, share of the step's kernel time,
DRAM bytes, GB/s) and merges per-profiling-kind DRAM traffic per launch into
profiles/traffic.json (the `roofline.traffic` bench.py reports).  ncu times are
cold-cache and serialised: compare shares, not absolutes.

usage: python tools/profile_summary.py launches.csv profiles/r01_launches_c2
"""
import collections
import csv
import json
import os
import sys

# kernel name -> library profiling kind (dt_profile_* kinds, csrc/prof.cu)
KIND = {
    "fused_kernel": "fused", "fused_small_kernel": "fused",
    "level_agg_kernel": "agg", "chunk_plan_kernel": "agg", "agg_scan_kernel": "agg",
    "piece_pos_kernel": "select", "select_kernel": "select",
    "number_kernel": "number", "children_kernel": "number", "tables_kernel": "number",
    "goleft_kernel": "goleft",
    "rs_count_kernel": "presort_sort", "rs_offset_kernel": "presort_sort", "rs_offset_warp_kernel": "presort_sort", "rs_scatter_kernel": "presort_sort",
    "root_reduce_kernel": "root_stats", "root_finalize_kernel": "root_stats", "root_center_kernel": "root_stats",
    "root_init_kernel": "root_stats", "root_tables_kernel": "presort_build",
    "predict_col_kernel": "predict", "eval_partial_kernel": "eval", "eval_final_kernel": "eval",
}


def short(name):
    base = name.split("(")[0]
    base = base.replace("dtl::<unnamed>::", "").replace("dtl::", "")
    if "DeviceRadixSort" in name or "cub::" in name:
        return "cub_radix_sort"
    if base.startswith("void "):
        base = base[5:]
    return base.split("<")[0]  # template arguments folded


def main():
    src, out = sys.argv[1], sys.argv[2]
    rows = list(csv.reader(open(src)))
    for i, r in enumerate(rows):
        if r and r[0] == "ID":
            hdr, start = r, i + 1
            break
    ki, mi, vi, idi = (hdr.index(k) for k in ("Kernel Name", "Metric Name", "Metric Value", "ID"))
    data = collections.OrderedDict()
    for r in rows[start:]:
        data.setdefault(r[idi], {"name": r[ki]})[r[mi]] = float(r[vi].replace(",", "") or 0)
    agg = collections.OrderedDict()
    for v in data.values():
        n = short(v["name"])
        a = agg.setdefault(n, [0, 0.0, 0.0])
        a[0] += 1
        a[1] += v.get("gpu__time_duration.sum", 0.0)
        a[2] += v.get("dram__bytes_read.sum", 0.0) + v.get("dram__bytes_write.sum", 0.0)
    nfit = max(1, agg.get("root_init_kernel", [1])[0])  # one root_init launch per fit
    for k in agg:
        agg[k] = [agg[k][0] / nfit, agg[k][1] / nfit, agg[k][2] / nfit]
    tot = sum(a[1] for a in agg.values())
    lines = [f"# ncu launch list: `{os.path.basename(src)}` (per fit; {nfit} fits captured)", "",
             "Cold-cache, serialised per-launch times (ncu `--clock-control none`); the bench's",
             "live CUDA-event times are the reference for absolutes. Share = fraction of the",
             "summed kernel time.", "",
             "| kernel | launches | time (us) | share | DRAM (MB) | GB/s |",
             "|---|---:|---:|---:|---:|---:|"]
    for n, (c, t, b) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"| {n} | {c:g} | {t / 1e3:.1f} | {t / tot:.3f} | {b / 1e6:.1f} | "
                     f"{(b / t if t else 0):.0f} |")
    lines.append(f"| **total** | {sum(a[0] for a in agg.values()):g} | {tot / 1e3:.1f} | 1.000 | | |")
    with open(out + ".md", "w") as fh:
        fh.write("\n".join(lines) + "\n")
    # traffic per launch of each profiling kind (a kind's launch = one library region)
    per_kind = collections.defaultdict(lambda: [0.0, 0])
    for n, (c, t, b) in agg.items():
        k = KIND.get(n)
        if k:
            per_kind[k][0] += b
    region_launches = {"fused": agg.get("fused_kernel", [1])[0],
                       "agg": agg.get("level_agg_kernel", [1])[0],
                       "select": agg.get("select_kernel", [1])[0],
                       "number": agg.get("number_kernel", [1])[0],
                       "goleft": agg.get("goleft_kernel", [1])[0],
                       "presort_sort": 1}
    tpath = os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "profiles", "traffic.json")
    traffic = {}  # this capture's kinds only
    for k, (b, _) in per_kind.items():
        launches = region_launches.get(k) or sum(c for n, (c, t, bb) in agg.items() if KIND.get(n) == k)
        traffic[k] = b / max(1, launches)
    traffic["_source"] = os.path.basename(src)
    with open(tpath, "w") as fh:
        json.dump(traffic, fh, indent=1, sort_keys=True)
    print("\n".join(lines))


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Summarise an `ncu --set full` capture exported with `--page raw --csv` (one row per
captured launch) into a markdown table: duration, DRAM bytes and throughput, SM / issue
activity, occupancy, registers, pipe utilisation and the top stall reasons.

usage: python tools/ncu_full_summary.py raw.csv out.md "title / command"
"""
import csv
import sys

COLS = [("duration (us)", "gpu__time_duration.sum", 1.0),
        ("DRAM read (MB)", "dram__bytes_read.sum", 1.0),
        ("DRAM write (MB)", "dram__bytes_write.sum", 1.0),
        ("DRAM % peak", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", 1.0),
        ("SM %", "sm__throughput.avg.pct_of_peak_sustained_elapsed", 1.0),
        ("issue active %", "sm__issue_active.avg.pct_of_peak_sustained_elapsed", 1.0),
        ("warps active %", "sm__warps_active.avg.pct_of_peak_sustained_active", 1.0),
        ("regs", "launch__registers_per_thread", 1.0),
        ("grid", "launch__grid_size", 1.0),
        ("block", "launch__block_size", 1.0),
        ("fp64 pipe %", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", 1.0),
        ("lsu pipe %", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", 1.0),
        ("warp instr (M)", "smsp__inst_executed.sum", 1e-6)]
STALLS = ["long_scoreboard", "short_scoreboard", "wait", "math_pipe_throttle", "mio_throttle",
          "lg_throttle", "barrier", "membar", "not_selected", "selected", "branch_resolving",
          "dispatch_stall", "no_instruction", "drain", "sleeping", "tex_throttle"]


def main():
    src, out, title = sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else ""
    rows = list(csv.reader(open(src)))
    hdr, units = rows[0], rows[1]
    idx = {h: i for i, h in enumerate(hdr)}

    def val(r, key, scale=1.0):
        i = idx.get(key)
        if i is None or not r[i]:
            return None
        try:
            v = float(r[i].replace(",", ""))
        except ValueError:
            return None
        u = units[i]
        if key.startswith("dram__bytes"):  # to MB
            v *= {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3}.get(u, 1.0)
        if key == "gpu__time_duration.sum":  # to us
            v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(u, 1.0)
        return v * scale

    lines = [f"# ncu --set full: {title}", "",
             "| kernel | " + " | ".join(c[0] for c in COLS) + " | top stalls (share of samples) |",
             "|---|" + "---:|" * len(COLS) + "---|"]
    for r in rows[2:]:
        name = r[idx["Kernel Name"]].split("(")[0].replace("unnamed>::", "").replace("void ", "")
        cells = []
        for _, key, sc in COLS:
            v = val(r, key, sc)
            cells.append("" if v is None else (f"{v:.0f}" if abs(v) >= 100 else f"{v:.2f}"))
        st = {}
        for s in STALLS:
            v = val(r, "smsp__pcsamp_warps_issue_stalled_" + s)
            if v:
                st[s] = v
        tot = sum(st.values()) or 1.0
        top = ", ".join(f"{k} {v / tot:.0%}" for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:4])
        lines.append(f"| {name} | " + " | ".join(cells) + f" | {top} |")
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()

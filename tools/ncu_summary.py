#!/usr/bin/env python
"""Summarise an .ncu-rep (raw page) into the metrics we track. usage: ncu_summary.py REP [REP...]"""
import csv
import io
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__cycles_elapsed.avg.per_second", "sm clock"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("dram__bytes_read.sum.per_second", "dram read BW"),
    ("smsp__inst_executed.sum", "warp instr"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "regs/thread"),
    ("launch__occupancy_limit_shared_mem", "CTA limit smem"),
    ("launch__occupancy_limit_registers", "CTA limit regs"),
    ("launch__grid_size", "grid"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "pipe alu %"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "pipe fma %"),
    ("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "pipe fp64 %"),
    ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "pipe xu %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "pipe lsu %"),
    ("sm__inst_executed_pipe_adu.avg.pct_of_peak_sustained_active", "pipe adu %"),
]
STALLS = "smsp__average_warps_issue_stalled_"


def summarise(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        out.append(f"== {path} :: {d.get('Kernel Name', '?')[:90]}")
        for k, name in KEYS:
            if k in d:
                out.append(f"  {name:24s} {d[k]} {u.get(k, '')}")
        st = [(k[len(STALLS):].replace("_per_issue_active.ratio", ""), float(v))
              for k, v in d.items() if k.startswith(STALLS) and k.endswith("per_issue_active.ratio")
              and v not in ("", "n/a")]
        st.sort(key=lambda x: -x[1])
        out.append("  stalls/issue: " + ", ".join(f"{n}={v:.2f}" for n, v in st[:8]))
    return "\n".join(out)


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(summarise(p))

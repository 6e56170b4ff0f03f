#!/usr/bin/env python
"""Top SASS instructions by a stall column from an ncu source page (sass view).
usage: ncu_src_stalls.py REP [COLUMN=stall_long_sb] [N=25]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
col = sys.argv[2] if len(sys.argv) > 2 else "stall_long_sb"
n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
lines = txt.splitlines()
rows = list(csv.reader(io.StringIO("\n".join(lines[1:]))))
hdr = rows[0]
ci = hdr.index(col)
si = hdr.index("Warp Stall Sampling (All Samples)")
tot = sum(float(r[si] or 0) for r in rows[1:] if len(r) > si)
totc = sum(float(r[ci] or 0) for r in rows[1:] if len(r) > ci)
print(f"total samples {tot:.0f}, {col} {totc:.0f} ({100 * totc / max(tot, 1):.1f}%)")
best = sorted(rows[1:], key=lambda r: -float(r[ci] or 0) if len(r) > ci else 0)[:n]
for r in best:
    print(f"{float(r[ci] or 0):8.0f}  {r[0]}  {r[1][:90]}")

#!/usr/bin/env python
"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into a markdown table.
usage: launches_md.py launches.csv [N]   (N: keep the first N launches of each kernel, e.g. the
bench steps before bench.py's K5 side reference)"""
import collections
import csv
import sys

lines = [l for l in open(sys.argv[1]).read().splitlines() if l.startswith('"')]
d = collections.OrderedDict()
for r in csv.DictReader(lines):
    if r["Metric Name"] != "gpu__time_duration.sum":
        continue
    k = r["Kernel Name"].split("(")[0]
    v = float(r["Metric Value"])
    unit = r.get("Metric Unit", "nsecond")
    v = v / 1e3 if unit.startswith("n") else v
    d.setdefault(k, []).append(v)
if len(sys.argv) > 2:
    n = int(sys.argv[2])
    d = collections.OrderedDict((k, v[:n]) for k, v in d.items())
tot = sum(sum(v) for v in d.values())
print("| kernel | launches | mean us | share of kernel time |")
print("|---|---|---|---|")
for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1])):
    print(f"| {k} | {len(v)} | {sum(v) / len(v):.1f} | {100 * sum(v) / tot:.1f}% |")

#!/usr/bin/env python
"""Print kernel name + metric values from `ncu --csv` output (stdin or file)."""
import csv
import sys

src = open(sys.argv[1]) if len(sys.argv) > 1 else sys.stdin
lines = [l for l in src.read().splitlines() if l.startswith('"')]
for r in csv.DictReader(lines):
    print(f'{r["Kernel Name"][:48]:48s} {r["Metric Name"]:28s} {r["Metric Value"]}')

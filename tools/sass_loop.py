#!/usr/bin/env python
"""Print / count the SASS of the hottest loop of a kernel in a .so (no GPU needed).

usage: sass_loop.py LIB FUNC_SUBSTR [--print]
Finds the backward branch whose body contains the most LDS.128 (the leaf
chain loop), then counts instructions per pipe class over the straight-line
fast path (branches to out-of-line slow paths are not followed).
"""
import re
import subprocess
import sys
from collections import Counter

lib, sub = sys.argv[1], sys.argv[2]
txt = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s*Function : ", txt)
body = None
for f in funcs:
    name = f.split("\n", 1)[0].strip()
    if sub in name:
        body = f
        fname = name
        break
if body is None:
    sys.exit(f"no function matching {sub}")
ins = []
for line in body.split("\n"):
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if m:
        ins.append((int(m.group(1), 16), m.group(2).strip()))
addr_idx = {a: i for i, (a, _) in enumerate(ins)}
best = None
for i, (a, t) in enumerate(ins):
    m = re.search(r"BRA(?:\.\S+)?\s+(?:!?U?P\d,\s*)?0x([0-9a-f]+)", t)
    if m:
        tgt = int(m.group(1), 16)
        if tgt < a and tgt in addr_idx:
            j = addr_idx[tgt]
            n_lds = sum(1 for _, x in ins[j:i + 1] if "LDS.128" in x)
            # innermost loop that holds a whole stage (>= 4 blocks) and issues its loads
            n_ld = sum(1 for _, x in ins[j:i + 1] if "LDGSTS" in x or "UTMALDG" in x)
            if n_lds >= 4 and n_ld > 0 and (best is None or i - j < best[1] - best[0]):
                best = (j, i, n_lds)
j, i, n_lds = best
loop = ins[j:i + 1]
# drop out-of-line slow paths: regions between 'BSSY' and 'BSYNC' that contain CALL
keep, buf, in_b = [], [], False
for a, t in loop:
    keep.append((a, t))
cls = Counter()
for a, t in keep:
    op = t.split()[0] if not t.startswith("@") else t.split()[1]
    cls[op.split(".")[0]] += 1
print(fname)
print(f"loop {loop[0][0]:#x}..{loop[-1][0]:#x}: {len(loop)} instr, {n_lds} LDS.128 -> {len(loop)/max(1,n_lds):.1f} per block (static, incl. slow-path stubs)")
print(" ".join(f"{k}:{v}" for k, v in cls.most_common()))
if "--print" in sys.argv:
    for a, t in loop:
        print(f"{a:#06x}  {t}")

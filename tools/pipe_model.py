#!/usr/bin/env python
"""Static pipe-cost model of the K1 hot loop (no GPU needed).

usage: pipe_model.py [-DFLAG ...]   (-DDTX=1: the f64 instantiation)
Compiles csrc/leaf.cuh's leaf_kernel<F32, !RAW, 4096, PAIR> alone to a cubin with the given
defines, finds the chain loop (as tools/sass_loop.py does) and prints per-16-byte-block
instruction counts and pipe cycles per SMSP under the rates measured on B200 with ncu
(profiles/r1_pipe_balance.md): fmaheavy IMAD 2 cycles, IMAD.WIDE 4; alu 2; issue 1.
"""
import os, re, subprocess, sys, tempfile
from collections import Counter

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_middleware_tanaabcrtn24_b200", "csrc")
defs = [a for a in sys.argv[1:] if a.startswith("-D")]
src = r'''
#ifndef DTX
#define DTX 0
#endif
#include "leaf.cuh"
template __global__ void ckpt::leaf_kernel<DTX, false, 4096, true, false>(const __grid_constant__ ckpt::LeafParams);
'''
with tempfile.TemporaryDirectory() as d:
    cu = os.path.join(d, "k.cu"); open(cu, "w").write(src)
    cub = os.path.join(d, "k.cubin")
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17",
                           "-cubin", "-I", CSRC, *defs, "-o", cub, cu])
    txt = subprocess.run(["cuobjdump", "-sass", cub], capture_output=True, text=True).stdout
ins = []
for line in txt.split("\n"):
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if m:
        ins.append((int(m.group(1), 16), m.group(2).strip()))
idx = {a: i for i, (a, _) in enumerate(ins)}
best = None
for i, (a, t) in enumerate(ins):
    m = re.search(r"BRA(?:\.\S+)?\s+(?:!?U?P\d,\s*)?0x([0-9a-f]+)", t)
    if m:
        tgt = int(m.group(1), 16)
        if tgt < a and tgt in idx:
            j = idx[tgt]
            nl = sum(1 for _, x in ins[j:i + 1] if "LDS.128" in x)
            ng = sum(1 for _, x in ins[j:i + 1] if "LDGSTS" in x)
            if nl >= 4 and ng > 0 and (best is None or i - j < best[1] - best[0]):
                best = (j, i, nl)
j, i, nb = best
ops = Counter()
for _, t in ins[j:i + 1]:
    t = re.sub(r"^@!?U?P\w+\s+", "", t)
    ops[t.split()[0]] += 1
fma = alu = 0.0
for op, n in ops.items():
    base = op.split(".")[0]
    if op.startswith("IMAD.WIDE"):
        fma += 4 * n
    elif base in ("IMAD", "IMUL"):
        fma += 2 * n
    elif base in ("IADD3", "LOP3", "SHF", "LEA", "FMNMX3", "FMNMX", "ISETP", "SEL", "PRMT", "MOV", "VIADD", "IABS", "FSETP", "PLOP3"):
        alu += 2 * n
tot = sum(ops.values())
print(f"{' '.join(defs) or '(default)'}: {tot/nb:.1f} instr/block  fmaheavy {fma/nb:.1f}  alu {alu/nb:.1f}  "
      f"bound {max(fma, alu, tot)/nb:.1f} cyc/block")
if "-v" in sys.argv:
    print(" ".join(f"{k}:{v/nb:.2f}" for k, v in ops.most_common()))

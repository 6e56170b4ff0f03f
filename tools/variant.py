#!/usr/bin/env python
"""Build an A/B variant of libckpt.so from a patched COPY of csrc/ (the product sources are not
touched): variants/<name>/libckpt.so.  Substitutions are exact text replacements that must match.

usage: variant.py NAME [FILE:OLD=>NEW ...]      (OLD/NEW: python string literals allowed via \\n)
Load a variant from a tool with  ck._lib = ck._declare(ctypes.CDLL(path))."""
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_middleware_tanaabcrtn24_b200 import _build  # noqa: E402


def build_variant(name, subs):
    vdir = os.path.join(ROOT, "variants", name)
    src = os.path.join(vdir, "csrc")
    if os.path.exists(src):
        shutil.rmtree(src)
    shutil.copytree(_build.CSRC, src)
    os.makedirs(os.path.join(vdir, "include"), exist_ok=True)
    shutil.copy(_build.HEADER, os.path.join(vdir, "include", "ckpt.h"))
    # csrc includes ../../include/ckpt.h: mirror the layout
    os.makedirs(os.path.join(vdir, "pkg"), exist_ok=True)
    for spec in subs:
        fname, rest = spec.split(":", 1)
        old, new = rest.split("=>", 1)
        old = old.encode().decode("unicode_escape")
        new = new.encode().decode("unicode_escape")
        p = os.path.join(src, fname)
        txt = open(p).read()
        if old not in txt:
            raise SystemExit(f"{name}: substitution not found in {fname}: {old[:80]!r}")
        open(p, "w").write(txt.replace(old, new))
    txt = open(os.path.join(src, "ckpt.cu")).read()
    open(os.path.join(src, "ckpt.cu"), "w").write(txt.replace('#include "../../include/ckpt.h"',
                                                              '#include "../include/ckpt.h"'))
    out = os.path.join(vdir, "libckpt.so")
    cmd = [_build._nvcc(), *_build.NVCC_FLAGS, "-o", out, os.path.join(src, "ckpt.cu")]
    subprocess.check_call(cmd)
    return out


if __name__ == "__main__":
    print(build_variant(sys.argv[1], sys.argv[2:]))

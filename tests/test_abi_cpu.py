"""CPU-side checks of the C-ABI boundary: libckpt.so loads and exports every declared symbol.

No compute entry point is called here (no GPU in this container)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ckpt.h")


def declared_functions():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    names = re.findall(r"\b(ckpt_[a-z0-9_]+)\s*\(", txt)
    return sorted(set(names))


@pytest.fixture(scope="module")
def libckpt():
    from paper_conf_middleware_tanaabcrtn24_b200 import _build
    _build.build()
    return ctypes.CDLL(_build.LIB)


def test_header_declares_the_north_star_calls():
    names = declared_functions()
    for required in ("ckpt_tree_build", "ckpt_tree_diff", "ckpt_verify", "ckpt_tree_free"):
        assert required in names


def test_every_declared_symbol_is_exported(libckpt):
    missing = [n for n in declared_functions() if not hasattr(libckpt, n)]
    assert not missing, missing


def test_status_strings_and_version(libckpt):
    libckpt.ckpt_strerror.restype = ctypes.c_char_p
    libckpt.ckpt_version.restype = ctypes.c_uint32
    assert libckpt.ckpt_strerror(0) == b"ok"
    assert libckpt.ckpt_strerror(-5).startswith(b"output truncated")
    assert libckpt.ckpt_version() >> 16 == 1


def test_library_is_sm100a_only():
    from paper_conf_middleware_tanaabcrtn24_b200 import _build
    assert "arch=compute_100a,code=sm_100a" in " ".join(_build.NVCC_FLAGS)


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_middleware_tanaabcrtn24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "ckpt_oracle" not in src and "liboracle" not in src, f

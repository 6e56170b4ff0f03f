"""CPU oracle for the error-bounded Merkle-tree checkpoint comparison path.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It never imports the product package
(``paper_conf_middleware_tanaabcrtn24_b200``) and the product never imports it.

The arithmetic lives in ``ckpt_oracle.c`` (plain C, one function per passage
of PAPER.md, see its header).  This module is argument marshalling (ctypes +
numpy) plus the per-array bookkeeping of a multi-array checkpoint:

* a checkpoint is an ordered list of arrays of one dtype (HACC writes one
  array per field per rank);
* each array gets its own Merkle tree (Alg. 1); the checkpoint
  root is the same level construction over the array roots (reading R15);
* chunk ids and element ids are global: array ``a``'s chunk ``c`` is
  ``chunk_base[a] + c`` and its element ``i`` is ``elem_base[a] + i``.

Parity status of every function: pinned.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass
from typing import List, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ckpt_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

F32 = 0
F64 = 1

CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
          "-pthread"]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (checker build, not product)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i64, u32, i32, dbl, vp = (ctypes.c_uint64, ctypes.c_int64, ctypes.c_uint32,
                                       ctypes.c_int, ctypes.c_double, ctypes.c_void_p)
        L.orc_murmur3f.argtypes = [vp, u64, u32, vp]
        L.orc_murmur3f_state.argtypes = [vp, u64, vp, vp]
        L.orc_quant_k.argtypes = [dbl, dbl]
        L.orc_quant_k.restype = i64
        L.orc_inv_eps.argtypes = [dbl]
        L.orc_inv_eps.restype = dbl
        L.orc_quantize.argtypes = [vp, u64, i32, dbl, vp]
        L.orc_n_chunks.argtypes = [u64, i32, u32]
        L.orc_n_chunks.restype = u64
        L.orc_leaves.argtypes = [vp, u64, i32, u32, dbl, i32, vp]
        L.orc_leaves.restype = i32
        L.orc_leaves_blk.argtypes = [vp, u64, i32, u32, dbl, u32, i32, vp]
        L.orc_leaves_blk.restype = i32
        L.orc_n_levels.argtypes = [u64]
        L.orc_n_levels.restype = u32
        L.orc_n_nodes.argtypes = [u64]
        L.orc_n_nodes.restype = u64
        L.orc_levels.argtypes = [vp, u64]
        L.orc_start_level.argtypes = [u64, u64]
        L.orc_start_level.restype = u32
        L.orc_diff.argtypes = [vp, vp, u64, u64, vp]
        L.orc_diff.restype = i64
        L.orc_verify.argtypes = [vp, vp, u64, i32, u32, vp, u64, dbl, vp, u64]
        L.orc_verify.restype = i64
        L.orc_brute.argtypes = [vp, vp, u64, i32, dbl, vp, u64]
        L.orc_brute.restype = i64
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def _dtype_code(a: np.ndarray) -> int:
    if a.dtype == np.float32:
        return F32
    if a.dtype == np.float64:
        return F64
    raise TypeError(f"oracle supports float32/float64, got {a.dtype}")


# --------------------------------------------------------------------------
# primitives
# --------------------------------------------------------------------------

def murmur3f(key: bytes, seed: int = 0) -> bytes:
    """SMHasher MurmurHash3_x64_128(key, len(key), seed) -> 16 bytes (h1||h2 LE)."""
    buf = np.frombuffer(bytes(key) + b"\0", dtype=np.uint8)
    out = np.zeros(16, np.uint8)
    lib().orc_murmur3f(_ptr(buf), len(key), seed, _ptr(out))
    return out.tobytes()


def murmur3f_state(key: bytes, h1: int, h2: int) -> tuple[int, int]:
    buf = np.frombuffer(bytes(key) + b"\0", dtype=np.uint8)
    a = ctypes.c_uint64(h1)
    b = ctypes.c_uint64(h2)
    lib().orc_murmur3f_state(_ptr(buf), len(key), ctypes.byref(a), ctypes.byref(b))
    return a.value, b.value


def inv_eps(eps: float) -> float:
    return lib().orc_inv_eps(eps)


def quant_k(x: float, eps: float) -> int:
    """k(x) = clamp(floor(x * RN(1/eps))) with NaN -> 0 (readings R5-R9)."""
    return lib().orc_quant_k(float(x), inv_eps(eps))


def quantize(a: np.ndarray, eps: float) -> np.ndarray:
    """Hashed words of every element (uint32 for f32, uint64 for f64)."""
    a = np.ascontiguousarray(a)
    out = np.empty(a.shape, np.uint32 if a.dtype == np.float32 else np.uint64)
    lib().orc_quantize(_ptr(a), a.size, _dtype_code(a), eps, _ptr(out))
    return out


def n_chunks(n: int, dtype_code: int, chunk_bytes: int) -> int:
    return lib().orc_n_chunks(n, dtype_code, chunk_bytes)


def leaves(a: np.ndarray, chunk_bytes: int, eps: float, threads: int = 1,
           hash_block: int = 16) -> np.ndarray:
    """(L, 16) uint8 leaf digests of one array (Alg. 1).

    hash_block: bytes per chained Murmur3F call (16 = the paper's 128-bit
    blocks; any multiple of 16; 0 = the whole chunk, R23)."""
    a = np.ascontiguousarray(a).reshape(-1)
    L = n_chunks(a.size, _dtype_code(a), chunk_bytes)
    out = np.zeros((L, 16), np.uint8)
    rc = lib().orc_leaves_blk(_ptr(a), a.size, _dtype_code(a), chunk_bytes, eps, hash_block,
                              threads, _ptr(out))
    if rc != 0:
        raise ValueError("invalid arguments to oracle leaves()")
    return out


def level_sizes(L: int) -> List[int]:
    s = [L]
    while s[-1] > 1:
        s.append((s[-1] + 1) // 2)
    return s


def levels(leaf_digests: np.ndarray) -> np.ndarray:
    """All tree nodes, leaf-first, root last: (n_nodes, 16) uint8 (Alg. 1)."""
    L = leaf_digests.shape[0]
    nodes = np.zeros((lib().orc_n_nodes(L), 16), np.uint8)
    nodes[:L] = leaf_digests
    lib().orc_levels(_ptr(nodes), L)
    return nodes


def start_level(L: int, T: int) -> int:
    return lib().orc_start_level(L, T)


def diff(nodes_a: np.ndarray, nodes_b: np.ndarray, L: int, T: int = 148 * 2048) -> np.ndarray:
    """Sorted differing chunk ids via the paper's BFS."""
    assert nodes_a.shape == nodes_b.shape
    out = np.zeros(L + 1, np.uint64)
    cnt = lib().orc_diff(_ptr(np.ascontiguousarray(nodes_a)), _ptr(np.ascontiguousarray(nodes_b)),
                         L, T, _ptr(out))
    return out[:cnt].astype(np.int64)


def verify(a: np.ndarray, b: np.ndarray, chunk_bytes: int, chunks: np.ndarray,
           eps: float) -> np.ndarray:
    """Sorted element ids i in the listed chunks with |a_i - b_i| > eps."""
    a = np.ascontiguousarray(a).reshape(-1)
    b = np.ascontiguousarray(b).reshape(-1)
    ch = np.ascontiguousarray(np.asarray(chunks, dtype=np.uint64))
    per = chunk_bytes // a.dtype.itemsize
    cap = max(1, ch.size * per)
    out = np.zeros(cap, np.uint64)
    cnt = lib().orc_verify(_ptr(a), _ptr(b), a.size, _dtype_code(a), chunk_bytes,
                           _ptr(ch) if ch.size else 0, ch.size, eps, _ptr(out), cap)
    return out[:cnt].astype(np.int64)


def brute(a: np.ndarray, b: np.ndarray, eps: float) -> np.ndarray:
    """Direct: sorted ids of every i with |a_i - b_i| > eps."""
    a = np.ascontiguousarray(a).reshape(-1)
    b = np.ascontiguousarray(b).reshape(-1)
    out = np.zeros(max(1, a.size), np.uint64)
    cnt = lib().orc_brute(_ptr(a), _ptr(b), a.size, _dtype_code(a), eps, _ptr(out), a.size)
    return out[:cnt].astype(np.int64)


# --------------------------------------------------------------------------
# multi-array checkpoints (per-array trees + top tree over roots, R15)
# --------------------------------------------------------------------------

@dataclass
class Checkpoint:
    trees: List[np.ndarray]       # per array: (n_nodes, 16) leaf-first
    n_leaves: List[int]
    top: np.ndarray               # tree over the array roots, leaf-first
    chunk_base: List[int]
    elem_base: List[int]

    @property
    def root(self) -> bytes:
        return self.top[-1].tobytes()

    @property
    def array_roots(self) -> np.ndarray:
        return np.stack([t[-1] for t in self.trees])


def build_checkpoint(arrays: Sequence[np.ndarray], chunk_bytes: int, eps: float,
                     threads: int = 1, hash_block: int = 16) -> Checkpoint:
    trees, nl, cb, eb = [], [], [], []
    c = e = 0
    for a in arrays:
        lv = leaves(a, chunk_bytes, eps, threads, hash_block)
        trees.append(levels(lv))
        nl.append(lv.shape[0])
        cb.append(c)
        eb.append(e)
        c += lv.shape[0]
        e += a.size
    top = levels(np.stack([t[-1] for t in trees]))
    return Checkpoint(trees, nl, top, cb, eb)


def diff_checkpoint(A: Checkpoint, B: Checkpoint, T: int = 148 * 2048) -> np.ndarray:
    out = [diff(ta, tb, L, T) + base
           for ta, tb, L, base in zip(A.trees, B.trees, A.n_leaves, A.chunk_base)]
    return np.concatenate(out) if out else np.zeros(0, np.int64)


def verify_checkpoint(arrays_a, arrays_b, chunk_bytes: int, chunks: np.ndarray, eps: float,
                      A: Checkpoint) -> np.ndarray:
    out = []
    chunks = np.asarray(chunks, np.int64)
    for k, (a, b) in enumerate(zip(arrays_a, arrays_b)):
        lo = A.chunk_base[k]
        hi = lo + A.n_leaves[k]
        mine = chunks[(chunks >= lo) & (chunks < hi)] - lo
        out.append(verify(a, b, chunk_bytes, mine, eps) + A.elem_base[k])
    return np.concatenate(out) if out else np.zeros(0, np.int64)


def brute_checkpoint(arrays_a, arrays_b, eps: float) -> np.ndarray:
    out, e = [], 0
    for a, b in zip(arrays_a, arrays_b):
        out.append(brute(a, b, eps) + e)
        e += a.size
    return np.concatenate(out) if out else np.zeros(0, np.int64)

"""Pure-Python second implementation of the oracle's encoding, for tiny inputs.

TEST INFRASTRUCTURE ONLY (same import rule as the ``oracle`` package).

Written independently of ``ckpt_oracle.c`` from the same definitions:

* ``murmur3f``: SMHasher MurmurHash3_x64_128 (footnote P:652).
* ``quant_k``: floor of the exact rational product x * RN(1/eps), clamped to
  int64, NaN -> 0 (readings R5-R9), evaluated with ``fractions.Fraction`` so
  no floating-point rounding enters after RN(1/eps).
* ``leaf``: Alg. 1 P:501-511 block chain with the full 128-bit digest as the
  next seed (R2) and a Murmur3F tail for a short final block (R12).
* ``levels``: Alg. 1 P:513-521 with odd-node promotion (R13).
"""
from __future__ import annotations

import math
import struct
from fractions import Fraction

M64 = (1 << 64) - 1
C1 = 0x87C37B91114253D5
C2 = 0x4CF5AD432745937F


def _rotl(x: int, r: int) -> int:
    return ((x << r) | (x >> (64 - r))) & M64


def _fmix(k: int) -> int:
    k ^= k >> 33
    k = (k * 0xFF51AFD7ED558CCD) & M64
    k ^= k >> 33
    k = (k * 0xC4CEB9FE1A85EC53) & M64
    k ^= k >> 33
    return k


def murmur3f_state(key: bytes, h1: int, h2: int) -> tuple[int, int]:
    n = len(key)
    nblocks = n // 16
    for i in range(nblocks):
        k1, k2 = struct.unpack_from("<QQ", key, 16 * i)
        k1 = (k1 * C1) & M64
        k1 = _rotl(k1, 31)
        k1 = (k1 * C2) & M64
        h1 ^= k1
        h1 = _rotl(h1, 27)
        h1 = (h1 + h2) & M64
        h1 = (h1 * 5 + 0x52DCE729) & M64
        k2 = (k2 * C2) & M64
        k2 = _rotl(k2, 33)
        k2 = (k2 * C1) & M64
        h2 ^= k2
        h2 = _rotl(h2, 31)
        h2 = (h2 + h1) & M64
        h2 = (h2 * 5 + 0x38495AB5) & M64
    tail = key[16 * nblocks:]
    rem = len(tail)
    if rem > 8:
        k2 = int.from_bytes(tail[8:], "little")
        k2 = (k2 * C2) & M64
        k2 = _rotl(k2, 33)
        k2 = (k2 * C1) & M64
        h2 ^= k2
    if rem > 0:
        k1 = int.from_bytes(tail[:8], "little")
        k1 = (k1 * C1) & M64
        k1 = _rotl(k1, 31)
        k1 = (k1 * C2) & M64
        h1 ^= k1
    h1 ^= n
    h2 ^= n
    h1 = (h1 + h2) & M64
    h2 = (h2 + h1) & M64
    h1 = _fmix(h1)
    h2 = _fmix(h2)
    h1 = (h1 + h2) & M64
    h2 = (h2 + h1) & M64
    return h1, h2


def murmur3f(key: bytes, seed: int = 0) -> bytes:
    h1, h2 = murmur3f_state(bytes(key), seed, seed)
    return struct.pack("<QQ", h1, h2)


def quant_k(x: float, eps: float) -> int:
    """floor(x * RN(1/eps)) in exact rational arithmetic, clamped; NaN -> 0."""
    if math.isnan(x):
        return 0
    inv = 1.0 / eps            # the one rounding the definition allows: RN(1/eps)
    if math.isinf(x):
        return (1 << 63) - 1 if x > 0 else -(1 << 63)
    k = math.floor(Fraction(x) * Fraction(inv))
    return max(-(1 << 63), min((1 << 63) - 1, k))


def words(values, is_f32: bool, eps: float) -> bytes:
    out = bytearray()
    for v in values:
        if eps == 0.0:
            out += struct.pack("<f" if is_f32 else "<d", v)
            continue
        k = quant_k(float(v), eps)
        if is_f32:
            out += struct.pack("<I", k & 0xFFFFFFFF)
        else:
            out += struct.pack("<Q", k & M64)
    return bytes(out)


def leaf(values, is_f32: bool, eps: float, block: int = 16) -> bytes:
    """block: hash block bytes (16 = P:610; 0 = the whole chunk)."""
    w = words(values, is_f32, eps)
    step = block if block else max(1, len(w))
    h1 = h2 = 0
    for off in range(0, len(w), step):
        h1, h2 = murmur3f_state(w[off:off + step], h1, h2)
    return struct.pack("<QQ", h1, h2)


def leaves(values, is_f32: bool, chunk_bytes: int, eps: float, block: int = 16) -> list[bytes]:
    per = chunk_bytes // (4 if is_f32 else 8)
    vals = list(values)
    return [leaf(vals[i:i + per], is_f32, eps, block) for i in range(0, len(vals), per)]


def levels(leaf_list: list[bytes]) -> list[list[bytes]]:
    lv = [list(leaf_list)]
    while len(lv[-1]) > 1:
        cur = lv[-1]
        nxt = []
        for j in range(0, len(cur), 2):
            if j + 1 < len(cur):
                nxt.append(murmur3f(cur[j] + cur[j + 1], 0))
            else:
                nxt.append(cur[j])
        lv.append(nxt)
    return lv

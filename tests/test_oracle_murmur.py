"""Pins for the oracle's Murmur3F (reading R1, footnote P:652)."""
import os
import re
import struct

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
from oracle import py_ref

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "smhasher_murmur3f.txt")


def _golden():
    txt = open(GOLDEN).read()
    ver = int(re.search(r"verification = (0x[0-9A-Fa-f]+)", txt).group(1), 16)
    empty = bytes.fromhex(re.search(r"empty_seed0 = ([0-9a-f]+)", txt).group(1))
    return ver, empty


def _smhasher_verification(h):
    key = bytes(range(256))
    hashes = b"".join(h(key[:i], 256 - i) for i in range(256))
    final = h(hashes, 0)
    return struct.unpack("<I", final[:4])[0]


def test_smhasher_verification_value_c_oracle():
    ver, _ = _golden()
    assert _smhasher_verification(oracle.murmur3f) == ver


def test_smhasher_verification_value_py_ref():
    ver, _ = _golden()
    assert _smhasher_verification(py_ref.murmur3f) == ver


def test_empty_input_seed0_is_zero():
    _, empty = _golden()
    assert oracle.murmur3f(b"", 0) == empty
    assert py_ref.murmur3f(b"", 0) == empty


@settings(max_examples=300, deadline=None)
@given(st.binary(min_size=0, max_size=80), st.integers(0, 2**32 - 1))
def test_c_matches_py_ref(key, seed):
    assert oracle.murmur3f(key, seed) == py_ref.murmur3f(key, seed)


@settings(max_examples=200, deadline=None)
@given(st.binary(min_size=0, max_size=40), st.integers(0, 2**64 - 1), st.integers(0, 2**64 - 1))
def test_state_seeded_matches_py_ref(key, h1, h2):
    assert oracle.murmur3f_state(key, h1, h2) == py_ref.murmur3f_state(key, h1, h2)


def test_state_api_with_equal_seeds_is_standard_api():
    rng = np.random.default_rng(0)
    for n in (0, 1, 7, 8, 9, 15, 16, 17, 31, 32, 33, 100):
        key = rng.integers(0, 256, n, dtype=np.uint8).tobytes()
        for seed in (0, 1, 0xDEADBEEF):
            h1, h2 = oracle.murmur3f_state(key, seed, seed)
            assert struct.pack("<QQ", h1, h2) == oracle.murmur3f(key, seed)


def test_single_bit_avalanche_sanity():
    # a correct finaliser flips ~half the 128 output bits for a 1-bit input change
    base = bytes(16)
    d0 = int.from_bytes(oracle.murmur3f(base), "little")
    flips = []
    for bit in range(128):
        k = bytearray(base)
        k[bit // 8] ^= 1 << (bit % 8)
        d1 = int.from_bytes(oracle.murmur3f(bytes(k)), "little")
        flips.append(bin(d0 ^ d1).count("1"))
    assert 50 < np.mean(flips) < 78

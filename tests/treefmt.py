"""Test-side writer of the serialised tree format documented in include/ckpt.h
("Tree persistence"), built from the ORACLE's trees -- an independent check
that the library reads and writes exactly the documented bytes.

Layout: "CKPTTRE1" | u32 1 | u32 dtype | u32 chunk_bytes | u32 hash_block |
f64 eps | u32 n_arrays | u32 0 | u64 n_elems[] | u64 node_count | root[16] |
nodes (level-major across arrays, then the top tree over the array roots).
"""
import struct

import numpy as np


def oracle_tree_bytes(ck, n_elems, dtype_code, chunk_bytes, eps, hash_block=16) -> bytes:
    """ck: oracle.Checkpoint.  hash_block: the effective block (16..chunk_bytes)."""
    na = len(ck.trees)
    sizes = []
    for L in ck.n_leaves:
        s = [L]
        while s[-1] > 1:
            s.append((s[-1] + 1) // 2)
        sizes.append(s)
    starts = [np.cumsum([0] + s[:-1]) for s in sizes]
    body = []
    for lvl in range(max(len(s) for s in sizes)):
        for a in range(na):
            if lvl < len(sizes[a]):
                o = starts[a][lvl]
                body.append(ck.trees[a][o:o + sizes[a][lvl]])
    body.append(ck.top)
    nodes = np.concatenate(body).astype(np.uint8)
    hdr = b"CKPTTRE1" + struct.pack("<IIIIdII", 1, dtype_code, chunk_bytes, hash_block, eps, na, 0)
    hdr += struct.pack(f"<{na}Q", *n_elems) + struct.pack("<Q", nodes.shape[0])
    return hdr + nodes[-1].tobytes() + nodes.tobytes()

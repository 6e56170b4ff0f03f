"""B200-native error-bounded Merkle-tree checkpoint comparison (Tan et al., MIDDLEWARE '24).

Thin ctypes binding over ``libckpt.so`` (C ABI in ``include/ckpt.h``).  This
module only marshals arguments (torch tensors -> device pointers, streams,
output buffers); every step of the path -- rounding + hashing, tree levels,
BFS diff, verification -- runs in the library's CUDA kernels.  There is no
CPU fallback: without the compiled library, or without a B200, every call
raises.

Function names follow the C ABI:

    tree_build(arrays, chunk_bytes, eps)      ckpt_tree_build_arrays   (Alg. 1)
    tree_diff(ta, tb)                         ckpt_tree_diff
    verify(a, b, chunks, chunk_bytes, eps)    ckpt_verify(_arrays)
    compare(arrays_a, arrays_b, ...)          ckpt_compare             (steps 1-4)
    compare_host(...)                         ckpt_compare_host        (host buffers)
    tree_from_digests(digests)                ckpt_tree_from_digests   (top tree, R15)
    tree_from_digests_batch(digests, counts)  ckpt_tree_from_digests_batch (several, one launch)
"""
from __future__ import annotations

import ctypes
import os
from typing import List, Optional, Sequence, Tuple, Union

import torch

from . import _build

__all__ = [
    "CkptError", "Tree", "lib", "tree_build", "tree_from_digests", "tree_diff", "tree_diff_async",
    "verify", "verify_async", "compare", "compare_host", "launch_count", "default_bfs_threshold",
    "tree_deserialize", "tree_load", "compare_saved", "compare_pair_async", "tree_build_batch",
    "compare_stream", "trim_device_memory",
    "F32", "F64",
]

F32 = 0
F64 = 1

OK, EINVAL, EMISMATCH, ENOMEM, ECUDA, ETRUNC = 0, -1, -2, -3, -4, -5


class CkptError(RuntimeError):
    def __init__(self, status: int, what: str):
        self.status = status
        super().__init__(f"{what}: status {status}")


_lib = None


def lib():
    """Load the in-tree libckpt.so.  Raises if it is missing: there is no fallback."""
    global _lib
    if _lib is not None:
        return _lib
    path = _build.LIB
    if not os.path.exists(path):
        raise ImportError(
            f"libckpt.so not built at {path}; run `python -c 'import __graft_entry__ as g; g.build()'`")
    _lib = _declare(ctypes.CDLL(path))
    return _lib


def _declare(L):
    """Argument and result types of the C ABI (include/ckpt.h)."""
    vp, u64, u32, i32, dbl = (ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int,
                              ctypes.c_double)
    pp = ctypes.POINTER(ctypes.c_void_p)
    pu64 = ctypes.POINTER(ctypes.c_uint64)
    L.ckpt_tree_build.argtypes = [vp, u64, i32, u32, dbl, vp, pp]
    L.ckpt_tree_build_arrays.argtypes = [pp, pu64, u32, i32, u32, dbl, vp, pp]
    L.ckpt_tree_build_batch.argtypes = [pp, pu64, ctypes.POINTER(u32), u32, i32, u32, dbl, vp, pp]
    L.ckpt_tree_build_batch_ex.argtypes = [pp, pu64, ctypes.POINTER(u32), u32, i32, u32, dbl, u32,
                                           vp, pp]
    L.ckpt_compare_pair_ex.argtypes = [pp, pp, pu64, u32, i32, u32, dbl, u32, vp, u64, vp, u64, vp,
                                       vp, pp, pp]
    L.ckpt_tree_serialized_size.argtypes = [vp, pu64]
    L.ckpt_tree_serialize.argtypes = [vp, vp, u64, pu64, vp]
    L.ckpt_tree_deserialize.argtypes = [vp, u64, vp, pp]
    L.ckpt_compare_saved.argtypes = [vp, u64, pp, pp, pu64, u32, vp, u64, vp, u64, vp, vp, pp, pp]
    L.ckpt_compare_stream.argtypes = [pp, pp, pu64, u32, i32, u32, dbl, u32, u64, vp, u64, vp, u64,
                                      pu64, pu64, vp, vp]
    L.ckpt_tree_params.argtypes = [vp, ctypes.POINTER(i32), ctypes.POINTER(u32),
                                   ctypes.POINTER(dbl), ctypes.POINTER(u32)]
    L.ckpt_tree_from_digests.argtypes = [vp, u64, vp, pp]
    L.ckpt_tree_from_digests_batch.argtypes = [vp, pu64, u32, vp, pp]
    L.ckpt_tree_free.argtypes = [vp]
    L.ckpt_tree_free.restype = None
    L.ckpt_tree_free_on.argtypes = [vp, vp]
    L.ckpt_tree_free_on.restype = None
    L.ckpt_tree_diff.argtypes = [vp, vp, vp, u64, pu64, vp]
    L.ckpt_tree_diff_async.argtypes = [vp, vp, u64, vp, u64, vp, vp]
    L.ckpt_verify.argtypes = [vp, vp, u64, i32, u32, vp, u64, dbl, vp, u64, pu64, vp]
    L.ckpt_verify_arrays_async.argtypes = [pp, pp, pu64, u32, i32, u32, vp, vp, u64, dbl, vp, u64,
                                           vp, vp]
    L.ckpt_compare.argtypes = [pp, pp, pu64, u32, i32, u32, dbl, vp, u64, vp, u64, pu64, pu64, vp,
                               vp, vp]
    L.ckpt_compare_host.argtypes = [pp, pp, pu64, u32, i32, u32, dbl, vp, u64, pu64, pu64, vp, vp]
    L.ckpt_tree_wait.argtypes = [vp, vp]
    L.ckpt_tree_info.argtypes = [vp, ctypes.POINTER(u32), pu64, ctypes.POINTER(u32), pu64]
    L.ckpt_tree_root.argtypes = [vp, vp, vp]
    L.ckpt_tree_array_roots.argtypes = [vp, vp, vp]
    L.ckpt_tree_nodes.argtypes = [vp, u32, vp, u64, vp]
    L.ckpt_tree_array_info.argtypes = [vp, u32, pu64, pu64]
    L.ckpt_profile_enable.argtypes = [i32]
    L.ckpt_profile_enable.restype = None
    L.ckpt_profile_reset.restype = None
    L.ckpt_profile_read.argtypes = [i32, ctypes.POINTER(dbl), pu64]
    L.ckpt_profile_read.restype = i32
    L.ckpt_profile_timeline.argtypes = [ctypes.POINTER(dbl), u64, pu64]
    L.ckpt_profile_timeline.restype = i32
    L.ckpt_default_bfs_threshold.restype = u64
    L.ckpt_launch_count.restype = u64
    L.ckpt_trim_device_memory.restype = i32
    L.ckpt_strerror.argtypes = [i32]
    L.ckpt_strerror.restype = ctypes.c_char_p
    L.ckpt_last_error.restype = ctypes.c_char_p
    L.ckpt_version.restype = u32
    for name in ("ckpt_tree_build", "ckpt_tree_build_arrays", "ckpt_tree_build_batch",
                 "ckpt_tree_build_batch_ex", "ckpt_compare_pair_ex", "ckpt_tree_params",
                 "ckpt_tree_serialized_size", "ckpt_tree_serialize", "ckpt_tree_deserialize",
                 "ckpt_compare_saved", "ckpt_compare_stream",
                 "ckpt_tree_from_digests", "ckpt_tree_from_digests_batch",
                 "ckpt_tree_diff", "ckpt_tree_diff_async", "ckpt_verify",
                 "ckpt_verify_arrays_async", "ckpt_compare", "ckpt_compare_host",
                 "ckpt_tree_info", "ckpt_tree_root", "ckpt_tree_array_roots", "ckpt_tree_nodes",
                 "ckpt_tree_array_info", "ckpt_tree_wait"):
        getattr(L, name).restype = i32
    return L


def _check(st: int, what: str, allow_trunc: bool = False):
    if st == OK or (allow_trunc and st == ETRUNC):
        return
    L = lib()
    msg = L.ckpt_last_error().decode(errors="replace")
    raise CkptError(st, f"{what}: {L.ckpt_strerror(st).decode()} ({msg})")


def _dtype_code(t: torch.Tensor) -> int:
    if t.dtype == torch.float32:
        return F32
    if t.dtype == torch.float64:
        return F64
    raise TypeError(f"only float32/float64 checkpoints are supported, got {t.dtype}")


def _stream_ptr(stream: Optional[torch.cuda.Stream]) -> int:
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


def _as_list(x) -> List[torch.Tensor]:
    if isinstance(x, torch.Tensor):
        return [x]
    return list(x)


def _check_arrays(arrays: Sequence[torch.Tensor]) -> int:
    if not arrays:
        raise ValueError("no arrays")
    code = _dtype_code(arrays[0])
    for t in arrays:
        if not t.is_cuda:
            raise ValueError("tensors must live on the CUDA device (use compare_host for host data)")
        if not t.is_contiguous():
            raise ValueError("tensors must be contiguous")
        if _dtype_code(t) != code:
            raise ValueError("all arrays of a checkpoint share one dtype")
    return code


def _check_out(t: torch.Tensor, what: str, min_numel: int = 0) -> None:
    """Output / device-count buffers handed to the kernels: int64, contiguous, on the current
    CUDA device, at least min_numel elements (numel() is passed as the capacity)."""
    if not isinstance(t, torch.Tensor) or t.dtype != torch.int64:
        raise TypeError(f"{what} must be an int64 tensor")
    if not t.is_cuda or t.device.index != torch.cuda.current_device():
        raise ValueError(f"{what} must live on the current CUDA device")
    if not t.is_contiguous():
        raise ValueError(f"{what} must be contiguous")
    if t.numel() < min_numel:
        raise ValueError(f"{what} needs at least {min_numel} elements")


def _ptr_array(ts: Sequence[torch.Tensor]):
    arr = (ctypes.c_void_p * len(ts))(*[t.data_ptr() for t in ts])
    return ctypes.cast(arr, ctypes.POINTER(ctypes.c_void_p)), arr


def _u64_array(vals: Sequence[int]):
    arr = (ctypes.c_uint64 * len(vals))(*vals)
    return ctypes.cast(arr, ctypes.POINTER(ctypes.c_uint64)), arr


class Tree:
    """Library-owned Merkle tree of one checkpoint (one or more arrays)."""

    def __init__(self, handle: int, arrays: Sequence[torch.Tensor], dtype: int, chunk_bytes: int,
                 eps: float, stream_ptr: int):
        self._h = ctypes.c_void_p(handle)
        self._keep = list(arrays)          # borrowed inputs must outlive the enqueued work
        self.dtype = dtype
        self.chunk_bytes = chunk_bytes
        self.eps = eps
        self._stream_ptr = stream_ptr
        na, nl = ctypes.c_uint32(), ctypes.c_uint64()
        nlev, nn = ctypes.c_uint32(), ctypes.c_uint64()
        _check(lib().ckpt_tree_info(self._h, ctypes.byref(na), ctypes.byref(nl), ctypes.byref(nlev),
                                    ctypes.byref(nn)), "ckpt_tree_info")
        self.n_arrays = na.value
        self.n_leaves = nl.value
        self.n_levels = nlev.value
        self.n_nodes = nn.value

    def detach_inputs(self) -> None:
        """Drop the references to the input arrays: call once the work that built the tree has
        completed on its stream (e.g. after a synchronize) to keep the tree without its data."""
        self._keep = []

    @property
    def handle(self):
        if self._h is None or not self._h.value:
            raise ValueError("tree already freed")
        return self._h

    def wait(self, stream=None):
        """Make `stream` wait until all levels are built (they build on a side stream)."""
        _check(lib().ckpt_tree_wait(self.handle, _stream_ptr(stream)), "ckpt_tree_wait")

    def root(self, stream=None) -> bytes:
        out = (ctypes.c_uint8 * 16)()
        _check(lib().ckpt_tree_root(self.handle, ctypes.cast(out, ctypes.c_void_p),
                                    _stream_ptr(stream)), "ckpt_tree_root")
        return bytes(out)

    def array_roots(self, stream=None, out: Optional[torch.Tensor] = None) -> torch.Tensor:
        """(n_arrays, 16) uint8 array roots; into `out` (a contiguous uint8 CUDA view) if given."""
        dst = out if out is not None else torch.empty((self.n_arrays, 16), dtype=torch.uint8,
                                                      device="cuda")
        if dst.dtype != torch.uint8 or not dst.is_contiguous() or dst.numel() != self.n_arrays * 16:
            raise ValueError("out must be a contiguous uint8 tensor of n_arrays x 16 bytes")
        _check(lib().ckpt_tree_array_roots(self.handle, dst.data_ptr(), _stream_ptr(stream)),
               "ckpt_tree_array_roots")
        return dst

    def params(self) -> Tuple[int, int, float, int]:
        """(dtype code, chunk_bytes, eps, effective hash block bytes) as stored in the tree."""
        d, c, e, h = ctypes.c_int(), ctypes.c_uint32(), ctypes.c_double(), ctypes.c_uint32()
        _check(lib().ckpt_tree_params(self.handle, ctypes.byref(d), ctypes.byref(c), ctypes.byref(e),
                                      ctypes.byref(h)), "ckpt_tree_params")
        return d.value, c.value, e.value, h.value

    def serialize(self, stream=None) -> bytes:
        """The tree in the documented on-disk format (ckpt_tree_serialize)."""
        n = ctypes.c_uint64()
        _check(lib().ckpt_tree_serialized_size(self.handle, ctypes.byref(n)), "ckpt_tree_serialized_size")
        buf = (ctypes.c_uint8 * n.value)()
        w = ctypes.c_uint64()
        _check(lib().ckpt_tree_serialize(self.handle, ctypes.cast(buf, ctypes.c_void_p), n.value,
                                         ctypes.byref(w), _stream_ptr(stream)), "ckpt_tree_serialize")
        return bytes(buf)

    def save(self, path: str, stream=None) -> None:
        with open(path, "wb") as f:
            f.write(self.serialize(stream))

    def array_info(self, array: int) -> Tuple[int, int]:
        nl, nn = ctypes.c_uint64(), ctypes.c_uint64()
        _check(lib().ckpt_tree_array_info(self.handle, array, ctypes.byref(nl), ctypes.byref(nn)),
               "ckpt_tree_array_info")
        return nl.value, nn.value

    def nodes(self, array: int = 0, stream=None) -> torch.Tensor:
        _, nn = self.array_info(array)
        dst = torch.empty((nn, 16), dtype=torch.uint8, device="cuda")
        _check(lib().ckpt_tree_nodes(self.handle, array, dst.data_ptr(), nn * 16,
                                     _stream_ptr(stream)), "ckpt_tree_nodes")
        return dst

    def free(self, stream=None):
        if self._h is not None and self._h.value:
            lib().ckpt_tree_free_on(self._h, _stream_ptr(stream) if stream is not None
                                    else self._stream_ptr)
        self._h = None
        self._keep = []

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def tree_build(arrays: Union[torch.Tensor, Sequence[torch.Tensor]], chunk_bytes: int, eps: float,
               stream=None, hash_block: int = 16) -> Tree:
    """Steps 1-2: leaves (quantize + chained Murmur3F) and all levels, asynchronously.

    hash_block: bytes per chained Murmur3F call (16 = P:610; 0 = whole chunk; R23)."""
    if hash_block != 16:
        return tree_build_batch([arrays], chunk_bytes, eps, stream, hash_block)[0]
    ts = _as_list(arrays)
    code = _check_arrays(ts)
    pp, _k1 = _ptr_array(ts)
    pn, _k2 = _u64_array([t.numel() for t in ts])
    out = ctypes.c_void_p()
    sp = _stream_ptr(stream)
    _check(lib().ckpt_tree_build_arrays(pp, pn, len(ts), code, chunk_bytes, float(eps), sp,
                                        ctypes.byref(out)), "ckpt_tree_build_arrays")
    return Tree(out.value, ts, code, chunk_bytes, float(eps), sp)


def tree_build_batch(checkpoints: Sequence[Sequence[torch.Tensor]], chunk_bytes: int, eps: float,
                     stream=None, hash_block: int = 16) -> List[Tree]:
    """Several checkpoints' trees with one leaf-kernel launch (ckpt_tree_build_batch[_ex])."""
    cks = [_as_list(c) for c in checkpoints]
    flat = [t for c in cks for t in c]
    code = _check_arrays(flat)
    pp, _k1 = _ptr_array(flat)
    pn, _k2 = _u64_array([t.numel() for t in flat])
    per = (ctypes.c_uint32 * len(cks))(*[len(c) for c in cks])
    outs = (ctypes.c_void_p * len(cks))()
    sp = _stream_ptr(stream)
    _check(lib().ckpt_tree_build_batch_ex(pp, pn, per, len(cks), code, chunk_bytes, float(eps),
                                          hash_block, sp,
                                          ctypes.cast(outs, ctypes.POINTER(ctypes.c_void_p))),
           "ckpt_tree_build_batch_ex")
    return [Tree(outs[k], cks[k], code, chunk_bytes, float(eps), sp) for k in range(len(cks))]


def tree_from_digests(digests: torch.Tensor, stream=None) -> Tree:
    """Tree whose leaves are the given (count, 16) uint8 digests (top tree over roots, R15)."""
    if digests.dtype != torch.uint8 or digests.dim() != 2 or digests.shape[1] != 16:
        raise ValueError("digests must be a (count, 16) uint8 tensor")
    d = digests.contiguous()
    out = ctypes.c_void_p()
    sp = _stream_ptr(stream)
    _check(lib().ckpt_tree_from_digests(d.data_ptr(), d.shape[0], sp, ctypes.byref(out)),
           "ckpt_tree_from_digests")
    return Tree(out.value, [d], F32, 16, 0.0, sp)


def tree_from_digests_batch(digests: torch.Tensor, counts: Sequence[int], stream=None) -> List[Tree]:
    """Several top trees with one levels launch: rows [sum(counts[:k]), +counts[k]) of the
    (sum(counts), 16) uint8 `digests` are the leaves of tree k."""
    if digests.dtype != torch.uint8 or digests.dim() != 2 or digests.shape[1] != 16:
        raise ValueError("digests must be a (count, 16) uint8 tensor")
    if sum(counts) != digests.shape[0]:
        raise ValueError("counts do not add up to the digest rows")
    d = digests.contiguous()
    n = len(counts)
    cnt = (ctypes.c_uint64 * n)(*[int(c) for c in counts])
    outs = (ctypes.c_void_p * n)()
    sp = _stream_ptr(stream)
    _check(lib().ckpt_tree_from_digests_batch(d.data_ptr(), cnt, n, sp, outs),
           "ckpt_tree_from_digests_batch")
    return [Tree(outs[k], [d], F32, 16, 0.0, sp) for k in range(n)]


def _host_blob(data):
    """(pointer, size) of a serialised tree given as bytes or a contiguous CPU uint8 tensor (pin it
    for a fast upload; bytes are copied into a ctypes buffer that lives as long as the call)."""
    if isinstance(data, torch.Tensor):
        if data.is_cuda or data.dtype != torch.uint8 or not data.is_contiguous():
            raise ValueError("a serialised tree tensor must be a contiguous CPU uint8 tensor")
        return ctypes.c_void_p(data.data_ptr()), data.numel()
    b = bytes(data)
    buf = ctypes.create_string_buffer(b, len(b))
    _host_blob.keep = buf
    return ctypes.cast(buf, ctypes.c_void_p), len(b)


def tree_deserialize(data, stream=None) -> Tree:
    """Load a serialised tree (bytes or CPU uint8 tensor) onto the current device."""
    buf, nbytes = _host_blob(data)
    out = ctypes.c_void_p()
    sp = _stream_ptr(stream)
    _check(lib().ckpt_tree_deserialize(buf, nbytes, sp, ctypes.byref(out)), "ckpt_tree_deserialize")
    t = Tree(out.value, [], F32, 0, 0.0, sp)
    t.dtype, t.chunk_bytes, t.eps, _ = t.params()
    return t


def tree_load(path: str, stream=None) -> Tree:
    with open(path, "rb") as f:
        return tree_deserialize(f.read(), stream)


def compare_saved(saved_a: bytes, arrays_a, arrays_b, chunks: torch.Tensor, idx: torch.Tensor,
                  counts: torch.Tensor, stream=None) -> Tuple[Tree, Tree]:
    """Compare live run B (device) with stored run A: A's tree from ``saved_a`` (serialised), A's
    data as device tensors or pinned host tensors (only flagged chunks are read), ckpt_compare_saved.

    Writes chunk ids, element ids and counts[0:2] (device) like compare_pair_async."""
    la, lb = _as_list(arrays_a), _as_list(arrays_b)
    if len(la) != len(lb) or any(x.numel() != y.numel() for x, y in zip(la, lb)):
        raise ValueError("A and B must have the same arrays and lengths")
    for t in la:
        if not t.is_cuda and not t.is_pinned():
            raise ValueError("host arrays of run A must be pinned (device-addressable)")
        if not t.is_contiguous():
            raise ValueError("arrays must be contiguous")
    code = _check_arrays(lb)
    _check_out(chunks, "chunks")
    _check_out(idx, "idx")
    _check_out(counts, "counts", 2)
    buf, nbytes = _host_blob(saved_a)
    hdr = ctypes.string_at(buf, 16) if nbytes >= 16 else b""
    if len(hdr) == 16 and int.from_bytes(hdr[12:16], "little") != code:
        raise ValueError("run B's dtype differs from the stored tree's")
    pa, _k1 = _ptr_array(la)
    pb, _k2 = _ptr_array(lb)
    pn, _k3 = _u64_array([t.numel() for t in lb])
    ta, tb = ctypes.c_void_p(), ctypes.c_void_p()
    sp = _stream_ptr(stream)
    _check(lib().ckpt_compare_saved(buf, nbytes, pa, pb, pn,
                                    len(lb), chunks.data_ptr(), chunks.numel(), idx.data_ptr(),
                                    idx.numel(), counts.data_ptr(), sp, ctypes.byref(ta),
                                    ctypes.byref(tb)), "ckpt_compare_saved")
    TA = Tree(ta.value, la, F32, 0, 0.0, sp)
    TA.dtype, TA.chunk_bytes, TA.eps, _ = TA.params()
    TB = Tree(tb.value, lb, TA.dtype, TA.chunk_bytes, TA.eps, sp)
    return TA, TB


def tree_diff(ta: Tree, tb: Tree, cap: Optional[int] = None, stream=None) -> torch.Tensor:
    """Step 3: ascending chunk ids whose leaves differ (BFS from the mid level)."""
    cap = ta.n_leaves if cap is None else cap
    out = torch.empty(max(cap, 1), dtype=torch.int64, device="cuda")
    n = ctypes.c_uint64()
    _check(lib().ckpt_tree_diff(ta.handle, tb.handle, out.data_ptr(), cap, ctypes.byref(n),
                                _stream_ptr(stream)), "ckpt_tree_diff", allow_trunc=True)
    return out[: min(n.value, cap)]


def tree_diff_async(ta: Tree, tb: Tree, chunks: torch.Tensor, count: torch.Tensor, T: int = 0,
                    stream=None):
    """Step 3 without a host round trip: count lands in count[0] on the device."""
    _check_out(chunks, "chunks")
    _check_out(count, "count", 1)
    _check(lib().ckpt_tree_diff_async(ta.handle, tb.handle, T, chunks.data_ptr(), chunks.numel(),
                                      count.data_ptr(), _stream_ptr(stream)), "ckpt_tree_diff_async")


def verify(a, b, chunks: torch.Tensor, chunk_bytes: int, eps: float, cap: Optional[int] = None,
           stream=None) -> Tuple[torch.Tensor, int]:
    """Step 4 on one array (sync): element ids with |a-b| > eps inside the listed chunks."""
    ta, tb = _as_list(a), _as_list(b)
    if len(ta) != 1:
        count = torch.zeros(2, dtype=torch.int64, device="cuda")
        count[0] = chunks.numel()
        out = torch.empty(max(cap or sum(t.numel() for t in ta), 1), dtype=torch.int64,
                          device="cuda")
        verify_async(ta, tb, chunks, count[0:1], chunk_bytes, eps, out, count[1:2], stream)
        n = int(count[1].item())
        return out[: min(n, out.numel())], n
    a, b = ta[0], tb[0]
    code = _check_arrays([a, b])
    ch = chunks.contiguous()
    cap = a.numel() if cap is None else cap
    out = torch.empty(max(cap, 1), dtype=torch.int64, device="cuda")
    n = ctypes.c_uint64()
    _check(lib().ckpt_verify(a.data_ptr(), b.data_ptr(), a.numel(), code, chunk_bytes,
                             ch.data_ptr() if ch.numel() else None, ch.numel(), float(eps),
                             out.data_ptr(), cap, ctypes.byref(n), _stream_ptr(stream)),
           "ckpt_verify", allow_trunc=True)
    return out[: min(n.value, cap)], n.value


def verify_async(arrays_a, arrays_b, chunks: torch.Tensor, n_chunks_dev: torch.Tensor,
                 chunk_bytes: int, eps: float, out: torch.Tensor, count_dev: torch.Tensor,
                 stream=None):
    """Step 4 over a multi-array checkpoint; chunk count read on the device."""
    ta, tb = _as_list(arrays_a), _as_list(arrays_b)
    code = _check_arrays(ta + tb)
    _check_out(chunks, "chunks")
    _check_out(n_chunks_dev, "n_chunks_dev", 1)
    _check_out(out, "out")
    _check_out(count_dev, "count_dev", 1)
    pa, _k1 = _ptr_array(ta)
    pb, _k2 = _ptr_array(tb)
    pn, _k3 = _u64_array([t.numel() for t in ta])
    _check(lib().ckpt_verify_arrays_async(pa, pb, pn, len(ta), code, chunk_bytes,
                                          chunks.data_ptr(), n_chunks_dev.data_ptr(),
                                          chunks.numel(), float(eps), out.data_ptr(), out.numel(),
                                          count_dev.data_ptr(), _stream_ptr(stream)),
           "ckpt_verify_arrays_async")


def compare(arrays_a, arrays_b, chunk_bytes: int, eps: float, chunks_cap: Optional[int] = None,
            idx_cap: Optional[int] = None, stream=None):
    """Steps 1-4 on device-resident checkpoints.

    Returns (chunks, idx, n_chunks, n_diff, root_a, root_b)."""
    ta, tb = _as_list(arrays_a), _as_list(arrays_b)
    code = _check_arrays(ta + tb)
    esz = 4 if code == F32 else 8
    L = sum(-(-t.numel() * esz // chunk_bytes) for t in ta)
    chunks_cap = L if chunks_cap is None else chunks_cap
    idx_cap = sum(t.numel() for t in ta) if idx_cap is None else idx_cap
    chunks = torch.empty(max(chunks_cap, 1), dtype=torch.int64, device="cuda")
    idx = torch.empty(max(idx_cap, 1), dtype=torch.int64, device="cuda")
    pa, _k1 = _ptr_array(ta)
    pb, _k2 = _ptr_array(tb)
    pn, _k3 = _u64_array([t.numel() for t in ta])
    nc, nd = ctypes.c_uint64(), ctypes.c_uint64()
    ra, rb = (ctypes.c_uint8 * 16)(), (ctypes.c_uint8 * 16)()
    _check(lib().ckpt_compare(pa, pb, pn, len(ta), code, chunk_bytes, float(eps),
                              chunks.data_ptr(), chunks_cap, idx.data_ptr(), idx_cap,
                              ctypes.byref(nc), ctypes.byref(nd), ctypes.cast(ra, ctypes.c_void_p),
                              ctypes.cast(rb, ctypes.c_void_p), _stream_ptr(stream)),
           "ckpt_compare", allow_trunc=True)
    return (chunks[: min(nc.value, chunks_cap)], idx[: min(nd.value, idx_cap)], nc.value,
            nd.value, bytes(ra), bytes(rb))


def compare_host(arrays_a, arrays_b, chunk_bytes: int, eps: float, idx_cap: Optional[int] = None):
    """Steps 1-4 on HOST checkpoints (pinned for speed); H2D/D2H inside the call.

    Returns (idx (host int64 tensor), n_chunks, n_diff, root_a, root_b)."""
    ta, tb = _as_list(arrays_a), _as_list(arrays_b)
    for t in ta + tb:
        if t.is_cuda or not t.is_contiguous():
            raise ValueError("compare_host takes contiguous host tensors")
    code = _dtype_code(ta[0])
    idx_cap = sum(t.numel() for t in ta) if idx_cap is None else idx_cap
    idx = torch.empty(max(idx_cap, 1), dtype=torch.int64)
    pa, _k1 = _ptr_array(ta)
    pb, _k2 = _ptr_array(tb)
    pn, _k3 = _u64_array([t.numel() for t in ta])
    nc, nd = ctypes.c_uint64(), ctypes.c_uint64()
    ra, rb = (ctypes.c_uint8 * 16)(), (ctypes.c_uint8 * 16)()
    _check(lib().ckpt_compare_host(pa, pb, pn, len(ta), code, chunk_bytes, float(eps),
                                   idx.data_ptr(), idx_cap, ctypes.byref(nc), ctypes.byref(nd),
                                   ctypes.cast(ra, ctypes.c_void_p),
                                   ctypes.cast(rb, ctypes.c_void_p)),
           "ckpt_compare_host", allow_trunc=True)
    return idx[: min(nd.value, idx_cap)], nc.value, nd.value, bytes(ra), bytes(rb)


def trim_device_memory() -> None:
    """Return the library's cached device memory to the driver (ckpt_trim_device_memory)."""
    _check(lib().ckpt_trim_device_memory(), "ckpt_trim_device_memory")


def compare_stream(arrays_a, arrays_b, chunk_bytes: int, eps: float,
                   segment_bytes: int = 256 << 20, hash_block: int = 16,
                   chunks_cap: Optional[int] = None, idx_cap: Optional[int] = None):
    """Steps 1-4 on HOST checkpoints streamed through a device ring (ckpt_compare_stream).

    Returns (chunks, idx (host int64 tensors), n_chunks, n_diff, root_a, root_b)."""
    ta, tb = _as_list(arrays_a), _as_list(arrays_b)
    if len(ta) != len(tb) or any(x.numel() != y.numel() for x, y in zip(ta, tb)):
        raise ValueError("A and B must have the same arrays and lengths")
    for t in ta + tb:
        if t.is_cuda or not t.is_contiguous():
            raise ValueError("compare_stream takes contiguous host tensors")
    code = _dtype_code(ta[0])
    esz = 4 if code == F32 else 8
    L = sum(-(-t.numel() * esz // chunk_bytes) for t in ta)
    chunks_cap = L if chunks_cap is None else chunks_cap
    idx_cap = sum(t.numel() for t in ta) if idx_cap is None else idx_cap
    chunks = torch.empty(max(chunks_cap, 1), dtype=torch.int64)
    idx = torch.empty(max(idx_cap, 1), dtype=torch.int64)
    pa, _k1 = _ptr_array(ta)
    pb, _k2 = _ptr_array(tb)
    pn, _k3 = _u64_array([t.numel() for t in ta])
    nc, nd = ctypes.c_uint64(), ctypes.c_uint64()
    ra, rb = (ctypes.c_uint8 * 16)(), (ctypes.c_uint8 * 16)()
    _check(lib().ckpt_compare_stream(pa, pb, pn, len(ta), code, chunk_bytes, float(eps), hash_block,
                                     segment_bytes, chunks.data_ptr(), chunks_cap, idx.data_ptr(),
                                     idx_cap, ctypes.byref(nc), ctypes.byref(nd),
                                     ctypes.cast(ra, ctypes.c_void_p),
                                     ctypes.cast(rb, ctypes.c_void_p)),
           "ckpt_compare_stream", allow_trunc=True)
    return (chunks[: min(nc.value, chunks_cap)], idx[: min(nd.value, idx_cap)], nc.value, nd.value,
            bytes(ra), bytes(rb))


def launch_count() -> int:
    return int(lib().ckpt_launch_count())


def default_bfs_threshold() -> int:
    return int(lib().ckpt_default_bfs_threshold())


KERNELS = {"leaf": 0, "levels": 1, "diff": 2, "verify": 3}


def profile_enable(on=True):
    """on: True (all kernel families), False, or a list of KERNELS names."""
    if on is True:
        mask = 0xF
    elif not on:
        mask = 0
    else:
        mask = 0
        for k in on:
            mask |= 1 << KERNELS[k]
    lib().ckpt_profile_enable(mask)


def profile_reset():
    lib().ckpt_profile_reset()


def profile_read(kernel: str) -> Tuple[float, int]:
    """(summed device ms, launches) of one kernel family since the last reset."""
    ms, n = ctypes.c_double(), ctypes.c_uint64()
    _check(lib().ckpt_profile_read(KERNELS[kernel], ctypes.byref(ms), ctypes.byref(n)),
           "ckpt_profile_read")
    return ms.value, n.value


def profile_timeline():
    """[(kernel, start_ms, end_ms)] of the recorded launches (relative to the first start)."""
    n = ctypes.c_uint64()
    _check(lib().ckpt_profile_timeline(None, 0, ctypes.byref(n)), "ckpt_profile_timeline")
    buf = (ctypes.c_double * (3 * max(n.value, 1)))()
    _check(lib().ckpt_profile_timeline(buf, n.value, ctypes.byref(n)), "ckpt_profile_timeline")
    names = {v: k for k, v in KERNELS.items()}
    return [(names.get(int(buf[3 * i]), "?"), buf[3 * i + 1], buf[3 * i + 2]) for i in range(n.value)]


def diff_verify_async(ta: Tree, tb: Tree, arrays_a, arrays_b, chunks: torch.Tensor,
                      idx: torch.Tensor, counts: torch.Tensor, stream=None):
    """Steps 3+4 in one call (one fused kernel when the BFS starts at the leaves).

    counts[0] / counts[1] (device int64) receive the flagged-chunk and differing-element counts."""
    ta_l, tb_l = _as_list(arrays_a), _as_list(arrays_b)
    _check_arrays(ta_l + tb_l)
    _check_out(chunks, "chunks")
    _check_out(idx, "idx")
    _check_out(counts, "counts", 2)
    pa, _k1 = _ptr_array(ta_l)
    pb, _k2 = _ptr_array(tb_l)
    L = lib()
    if not getattr(L, "_dv_typed", False):
        L.ckpt_diff_verify_async.argtypes = [ctypes.c_void_p, ctypes.c_void_p,
                                             ctypes.POINTER(ctypes.c_void_p),
                                             ctypes.POINTER(ctypes.c_void_p), ctypes.c_void_p,
                                             ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint64,
                                             ctypes.c_void_p, ctypes.c_void_p]
        L.ckpt_diff_verify_async.restype = ctypes.c_int
        L._dv_typed = True
    _check(L.ckpt_diff_verify_async(ta.handle, tb.handle, pa, pb, chunks.data_ptr(), chunks.numel(),
                                    idx.data_ptr(), idx.numel(), counts.data_ptr(),
                                    _stream_ptr(stream)), "ckpt_diff_verify_async")


def compare_pair_async(arrays_a, arrays_b, chunk_bytes: int, eps: float, chunks: torch.Tensor,
                       idx: torch.Tensor, counts: torch.Tensor, stream=None,
                       hash_block: int = 16) -> Tuple[Tree, Tree]:
    """Fused pair compare (ckpt_compare_pair_async): steps 1-4 for two checkpoints of identical
    shape with the leaf-digest comparison and the element marking inside the leaf kernel.

    Writes the flagged chunk ids to ``chunks``, the differing element ids to ``idx`` and the two
    full counts to ``counts[0:2]`` (device int64); returns both trees."""
    la, lb = _as_list(arrays_a), _as_list(arrays_b)
    if len(la) != len(lb) or any(x.numel() != y.numel() for x, y in zip(la, lb)):
        raise ValueError("A and B must have the same arrays and lengths")
    code = _check_arrays(la + lb)
    _check_out(chunks, "chunks")
    _check_out(idx, "idx")
    _check_out(counts, "counts", 2)
    pa, _k1 = _ptr_array(la)
    pb, _k2 = _ptr_array(lb)
    pn, _k3 = _u64_array([t.numel() for t in la])
    ta, tb = ctypes.c_void_p(), ctypes.c_void_p()
    sp = _stream_ptr(stream)
    _check(lib().ckpt_compare_pair_ex(pa, pb, pn, len(la), code, chunk_bytes, float(eps), hash_block,
                                      chunks.data_ptr(), chunks.numel(), idx.data_ptr(), idx.numel(),
                                      counts.data_ptr(), sp, ctypes.byref(ta), ctypes.byref(tb)),
           "ckpt_compare_pair_ex")
    return (Tree(ta.value, la, code, chunk_bytes, float(eps), sp),
            Tree(tb.value, lb, code, chunk_bytes, float(eps), sp))

"""Seeded synthetic checkpoint generator shared by the tests, the bench and smoke().

This module holds NONE of the method's arithmetic (no quantizer, no hash, no
difference predicate).  It only draws HACC-shaped inputs (Table 1,
P:745-761: per-particle x, y, z, vx, vy, vz as float32) and injects
perturbations of intended sizes; the expected outputs always come from the
oracle run on the stored bytes.

RNG: counter-based splitmix64(seed, index) in int64 torch ops, so the same
(seed, index) gives the same uniform bits on CPU and GPU.  Normals use
Box-Muller (transcendentals may differ in the last bit between devices,
which is harmless: both sides of every parity test read the same stored
bytes).

Recipes:
  c1  2^20 f32 ~ U[-1,1), eps 1e-5, C 4 KiB; run B = A + 100 perturbations at
      distinct indices: 50 "above" |d| ~ U[2,20]*eps, 50 "below" |d| ~
      U[0.05,0.5]*eps of which >= 10 straddle a multiple of eps.
  c2  2^26 particles x 6 f32 SoA arrays: x,y,z ~ U[0,256), v* ~ N(0, 300^2);
      eps 1e-6, C 4 KiB; 1% of particles in 64 contiguous clusters get
      d = +-10^U(-8,-3) on all six fields.
  c3  2^29 f64 ~ N(0,1); 1024 clusters, geometric length (mean 4096),
      d = +-10^U(-9,-2); plus 2^16 isolated d = +-10^U(-10,-1) (eps-dependent
      flagging and false positives across the sweep).
  c4  per-rank c2-shaped arrays (rank_pair).
  c5  8 ranks x 50*2^20 particles x 6 f32 per GPU; 10% of chunks get 8 above-eps
      and 8 below-eps (bin-straddling) perturbations, another 1% only the
      below-eps ones (verify-heavy, false positives by construction).
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import List

import numpy as np
import torch

_GOLDEN = -7046029254386353131      # 0x9E3779B97F4A7C15 as int64
_M1 = -4658895280553007687          # 0xBF58476D1CE4E5B9
_M2 = -7723592293110705685          # 0x94D049BB133111EB


def _srl(z: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (z >> s) & ((1 << (64 - s)) - 1)


def splitmix64(seed: int, idx: torch.Tensor) -> torch.Tensor:
    """splitmix64 output for counters idx (int64 tensor) under `seed`."""
    s = (seed * 0x632BE59BD9B4E019) & ((1 << 64) - 1)
    if s >= 1 << 63:
        s -= 1 << 64
    z = idx.to(torch.int64) * _GOLDEN + s
    z = z + _GOLDEN
    z = (z ^ _srl(z, 30)) * _M1
    z = (z ^ _srl(z, 27)) * _M2
    return z ^ _srl(z, 31)


def _arange(n: int, offset: int, device) -> torch.Tensor:
    return torch.arange(offset, offset + n, dtype=torch.int64, device=device)


def uniform(seed: int, n: int, device="cpu", offset: int = 0, dtype=torch.float32) -> torch.Tensor:
    """U[0,1) with 24 (f32) or 53 (f64) random bits; exact on every device."""
    z = splitmix64(seed, _arange(n, offset, device))
    if dtype == torch.float32:
        return _srl(z, 40).to(torch.float32) * (2.0 ** -24)
    return _srl(z, 11).to(torch.float64) * (2.0 ** -53)


def normal(seed: int, n: int, device="cpu", offset: int = 0, dtype=torch.float32) -> torch.Tensor:
    """N(0,1) by Box-Muller from two counter streams (computed in f64)."""
    u1 = uniform(seed, n, device, offset, torch.float64)
    u2 = uniform(seed ^ 0x5DEECE66D, n, device, offset, torch.float64)
    r = torch.sqrt(-2.0 * torch.log1p(-u1))
    out = r * torch.cos(2.0 * np.pi * u2)
    return out.to(dtype)


# --------------------------------------------------------------------------
# checkpoint pairs
# --------------------------------------------------------------------------

@dataclass
class Pair:
    name: str
    a: List[torch.Tensor]             # run A arrays
    b: List[torch.Tensor]             # run B arrays
    chunk_bytes: int
    eps: float
    meta: dict = field(default_factory=dict)

    @property
    def nbytes(self) -> int:
        return sum(t.numel() * t.element_size() for t in self.a)


def c1_pair(n: int = 1 << 20, seed: int = 1, device="cpu", eps: float = 1e-5,
            chunk_bytes: int = 4096, n_above: int = 50, n_below: int = 50,
            n_straddle: int = 10) -> Pair:
    """Config 1: U[-1,1) f32 with 100 injected perturbations (BASELINE configs[0])."""
    a = uniform(seed, n, device) * 2.0 - 1.0
    b = a.clone()
    rng = np.random.default_rng(seed)
    k = n_above + n_below
    idx = rng.choice(n, size=min(k, n), replace=False)
    sign = np.where(rng.random(idx.size) < 0.5, -1.0, 1.0)
    mag = np.empty(idx.size)
    na = min(n_above, idx.size)
    mag[:na] = rng.uniform(2.0, 20.0, na) * eps
    mag[na:] = rng.uniform(0.05, 0.5, idx.size - na) * eps
    a_np = a.cpu().numpy().astype(np.float64)
    vals_a = a_np[idx].copy()
    vals_b = vals_a + sign * mag
    # straddlers: a just below a multiple of eps, b just above (false positives)
    ns = min(n_straddle, idx.size - na)
    for q in range(na, na + ns):
        m = np.round(vals_a[q] / eps)
        off = rng.uniform(0.02, 0.2) * eps
        vals_a[q] = m * eps - off
        vals_b[q] = m * eps + off
    ia = torch.as_tensor(idx, dtype=torch.int64, device=device)
    a[ia] = torch.as_tensor(vals_a, dtype=torch.float32, device=device)
    b[ia] = torch.as_tensor(vals_b, dtype=torch.float32, device=device)
    return Pair("c1", [a], [b], chunk_bytes, eps,
                {"n": n, "perturbed": idx, "n_above": na, "n_straddle": ns})


HACC_FIELDS = ("x", "y", "z", "vx", "vy", "vz")


def hacc_arrays(n_particles: int, seed: int, device="cpu", box: float = 256.0,
                vsigma: float = 300.0) -> List[torch.Tensor]:
    """Six SoA float32 arrays shaped like a HACC checkpoint (Table 1)."""
    out = []
    for f in range(6):
        s = seed * 16 + f
        if f < 3:
            out.append(uniform(s, n_particles, device) * box)
        else:
            out.append(normal(s, n_particles, device) * vsigma)
    return out


def cluster_mask_perturb(arrays: List[torch.Tensor], frac: float, n_clusters: int, seed: int,
                         lo_exp: float = -8.0, hi_exp: float = -3.0) -> tuple:
    """Copy `arrays` and add d = +-10^U(lo,hi) to `frac` of the indices, laid out as
    `n_clusters` contiguous clusters (same indices in every array)."""
    n = arrays[0].numel()
    device = arrays[0].device
    rng = np.random.default_rng(seed)
    total = int(round(frac * n))
    starts, lens = [], []
    if total > 0 and n_clusters > 0:
        per = max(1, total // n_clusters)
        cand = np.sort(rng.choice(max(1, n - per), size=n_clusters, replace=False))
        for s in cand:
            starts.append(int(s))
            lens.append(per)
    out = [t.clone() for t in arrays]
    for f, t in enumerate(out):
        for c, (s, ln) in enumerate(zip(starts, lens)):
            sub = torch.arange(s, s + ln, device=device, dtype=torch.int64)
            u = uniform(seed * 977 + f * 131 + c, ln, device, dtype=torch.float64)
            sg = uniform(seed * 1931 + f * 17 + c, ln, device, dtype=torch.float64)
            d = torch.pow(10.0, lo_exp + (hi_exp - lo_exp) * u) * torch.where(sg < 0.5, -1.0, 1.0)
            t[sub] = (t[sub].to(torch.float64) + d).to(t.dtype)
    return out, list(zip(starts, lens))


def c2_pair(n_particles: int = 1 << 26, seed: int = 2, device="cpu", eps: float = 1e-6,
            chunk_bytes: int = 4096, frac: float = 0.01, n_clusters: int = 64) -> Pair:
    """Config 2: HACC-shaped 6 x f32 per GPU, clustered divergence (BASELINE configs[1])."""
    a = hacc_arrays(n_particles, seed, device)
    b, clusters = cluster_mask_perturb(a, frac, n_clusters, seed + 1000)
    return Pair("c2", a, b, chunk_bytes, eps,
                {"n_particles": n_particles, "clusters": clusters})


def c3_pair(n: int = 1 << 29, seed: int = 3, device="cpu", eps: float = 1e-6,
            chunk_bytes: int = 4096, n_clusters: int = 1024, mean_len: int = 4096,
            n_isolated: int = 1 << 16, iso_exp=(-10.0, -1.0)) -> Pair:
    """Config 3: N(0,1) f64 with geometric-length clustered divergence plus `n_isolated`
    single-element changes of log-uniform size 10^U(iso_exp) at uniform random indices: around
    any eps of the sweep some of them exceed eps (true positives) and some smaller ones straddle
    a bin edge (false positives), so the flagged fraction and the false-positive rate depend on
    eps (the synthetic analogue of Fig. 7)."""
    a = normal(seed, n, device, dtype=torch.float64)
    b = a.clone()
    rng = np.random.default_rng(seed)
    starts = rng.integers(0, n, size=n_clusters)
    lens = rng.geometric(1.0 / mean_len, size=n_clusters)
    for c, (s, ln) in enumerate(zip(starts, lens)):
        ln = int(min(ln, n - s))
        sub = torch.arange(int(s), int(s) + ln, device=device, dtype=torch.int64)
        u = uniform(seed * 7919 + c, ln, device, dtype=torch.float64)
        sg = uniform(seed * 104729 + c, ln, device, dtype=torch.float64)
        d = torch.pow(10.0, -9.0 + 7.0 * u) * torch.where(sg < 0.5, -1.0, 1.0)
        b[sub] = b[sub] + d
    if n_isolated > 0:
        iso = torch.as_tensor(np.unique(rng.integers(0, n, size=n_isolated)), dtype=torch.int64,
                              device=device)
        m = iso.numel()
        u = uniform(seed * 31337 + 1, m, device, dtype=torch.float64)
        sg = uniform(seed * 31337 + 2, m, device, dtype=torch.float64)
        lo, hi = iso_exp
        d = torch.pow(10.0, lo + (hi - lo) * u) * torch.where(sg < 0.5, -1.0, 1.0)
        b[iso] = b[iso] + d
    return Pair("c3", [a], [b], chunk_bytes, eps, {"n": n, "n_isolated": n_isolated})


def rank_pair(rank: int, n_particles: int, seed_base: int, device="cpu", eps: float = 1e-6,
              chunk_bytes: int = 4096, frac: float = 0.01, n_clusters: int = 8) -> Pair:
    """One HACC rank's checkpoint pair (c4/c5 shards): 6 f32 arrays per run."""
    a = hacc_arrays(n_particles, seed_base + rank, device)
    b, clusters = cluster_mask_perturb(a, frac, n_clusters, seed_base + 5000 + rank)
    return Pair(f"rank{rank}", a, b, chunk_bytes, eps, {"clusters": clusters})


def c4_frac(snapshot: int) -> float:
    """Config 4 divergence: none for s <= 2, then 1e-6 * 4^(s-3) of the particles."""
    return 0.0 if snapshot <= 2 else 1e-6 * 4.0 ** (snapshot - 3)


def c4_snapshot(snapshot: int, ranks, n_particles: int = 1 << 24, device="cpu",
                eps: float = 1e-6, chunk_bytes: int = 4096, n_clusters: int = 8) -> Pair:
    """Config 4 (BASELINE configs[3]): one intermediate snapshot of a 64-rank HACC run, the
    given ranks only (a GPU's shard): 6 f32 arrays per rank per run, 2^24 particles per rank
    (2^30 in total), clustered divergence growing with the snapshot index (c4_frac)."""
    frac = c4_frac(snapshot)
    a_list, b_list, meta = [], [], {}
    for r in ranks:
        a = hacc_arrays(n_particles, (40 + snapshot) * 1000 + r, device)
        if frac > 0:
            b, cl = cluster_mask_perturb(a, frac, n_clusters, (40 + snapshot) * 1000 + 500 + r)
        else:
            b, cl = [t.clone() for t in a], []
        a_list += a
        b_list += b
        meta[r] = cl
    return Pair(f"c4_s{snapshot}", a_list, b_list, chunk_bytes, eps,
                {"snapshot": snapshot, "ranks": list(ranks), "frac": frac, "clusters": meta})


def c5_pair(n_ranks: int = 8, n_particles: int = 50 << 20, seed: int = 50, device="cpu",
            eps: float = 1e-6, chunk_bytes: int = 4096, frac_true: float = 0.10,
            frac_fp: float = 0.01, per_chunk: int = 8) -> Pair:
    """Config 5 (per GPU): n_ranks HACC ranks x 6 f32 arrays per run.

    In frac_true of the chunks of every array, `per_chunk` elements get
    |d| ~ U[2,20]*eps (above) and `per_chunk` more straddle a multiple of eps
    at a small magnitude (below, forced false positive); in another frac_fp of
    the chunks only the straddlers are planted.  Straddling changes run A too
    (a = m*eps - off, b = m*eps + off with off < eps/2)."""
    a_list, b_list = [], []
    rng = np.random.default_rng(seed)
    per = chunk_bytes // 4
    for r in range(n_ranks):
        arrs = hacc_arrays(n_particles, seed * 100 + r, device)
        outs = [t.clone() for t in arrs]
        for f, (ta, tb) in enumerate(zip(arrs, outs)):
            n = ta.numel()
            L = n // per
            n_true = int(round(frac_true * L))
            n_fp = int(round(frac_fp * L))
            ch = rng.choice(L, size=n_true + n_fp, replace=False)
            ch_true, ch_fp = ch[:n_true], ch[n_true:]
            # above-eps: per_chunk random elements of each true chunk
            if n_true:
                off = rng.integers(0, per, size=(n_true, per_chunk))
                idx = (ch_true[:, None] * per + off).reshape(-1)
                idx = np.unique(idx)
                sgn = np.where(rng.random(idx.size) < 0.5, -1.0, 1.0)
                mag = rng.uniform(2.0, 20.0, idx.size) * eps * sgn
                it = torch.as_tensor(idx, dtype=torch.int64, device=device)
                x = tb[it].to(torch.float64)
                md = torch.as_tensor(mag, device=device)
                # at least ~2 ulps of x so the change survives rounding to f32
                md = torch.sign(md) * torch.maximum(md.abs(), x.abs() * 2.0 ** -22)
                tb[it] = (x + md).to(tb.dtype)
            # below-eps bin straddlers in true and fp chunks
            chs = np.concatenate([ch_true, ch_fp])
            if chs.size:
                off = rng.integers(0, per, size=(chs.size, per_chunk))
                idx = np.unique((chs[:, None] * per + off).reshape(-1))
                m = rng.integers(-500, 500, idx.size).astype(np.float64)
                d = rng.uniform(0.02, 0.2, idx.size) * eps
                va = torch.as_tensor(m * eps - d, dtype=torch.float32, device=device)
                vb = torch.as_tensor(m * eps + d, dtype=torch.float32, device=device)
                it = torch.as_tensor(idx, dtype=torch.int64, device=device)
                ta[it] = va
                tb[it] = vb
        a_list += arrs
        b_list += outs
    return Pair("c5", a_list, b_list, chunk_bytes, eps,
                {"n_ranks": n_ranks, "n_particles": n_particles})

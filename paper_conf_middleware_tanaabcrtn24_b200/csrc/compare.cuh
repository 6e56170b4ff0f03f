// compare.cuh -- K3 (BFS diff, P:555-566 / P:642-648) and K4 (verify).
//
// Both emit unique ascending ids (reading R17) with a single-pass ordered
// compaction: each CTA takes tiles in order from an atomic ticket, counts its
// hits with __ballot_sync/__popc, publishes the tile aggregate and looks back
// over its predecessors (decoupled look-back) for its exclusive prefix, then
// writes its hits at their final positions.  Persistent grids, so the item
// counts may live on the device (no host round trip between steps).
#pragma once
#include <cstdint>

#include "hash.cuh"

namespace ckpt {

constexpr unsigned kFull = 0xffffffffu;
// Look-back state word: epoch (24 bits) | flag (2 bits) | value (38 bits).
// The epoch is new for every launch that uses a scratch buffer, so states left
// by earlier launches read as "not ready" and the buffer never needs clearing.
constexpr int kValBits = 38;
constexpr uint64_t kValMask = (1ull << kValBits) - 1;
constexpr uint64_t kFlagA = 1ull << kValBits;        // tile aggregate available
constexpr uint64_t kFlagP = 2ull << kValBits;        // inclusive prefix available

__device__ __forceinline__ uint64_t ld_volatile(const uint64_t *p) {
    return *reinterpret_cast<const volatile uint64_t *>(p);
}
__device__ __forceinline__ void st_volatile(uint64_t *p, uint64_t v) {
    *reinterpret_cast<volatile uint64_t *>(p) = v;
}
__device__ __forceinline__ uint64_t state_word(uint32_t epoch, uint64_t flag, uint64_t v) {
    return ((uint64_t)epoch << 40) | flag | (v & kValMask);
}

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return v;
}

__device__ __forceinline__ uint32_t warp_excl_scan_u32(uint32_t v, int lane, uint32_t &total) {
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= o) x += y;
    }
    total = __shfl_sync(kFull, x, 31);
    return x - v;
}

// CTA-wide decoupled look-back: every thread inspects one predecessor per
// round, so a round covers blockDim.x predecessors with one L2 round trip.
// Called by all threads; `aggregate` must be the same in every thread.
// Returns the tile's exclusive prefix.
template <int NT>
__device__ uint64_t cta_lookback(uint64_t *states, uint64_t tile, uint64_t aggregate, uint32_t epoch) {
    constexpr int NW = NT / 32;
    __shared__ uint64_t s_sum[NW];
    __shared__ int s_min[NW];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tile == 0) {
        if (tid == 0) st_volatile(&states[0], state_word(epoch, kFlagP, aggregate));
        return 0;
    }
    if (tid == 0) st_volatile(&states[tile], state_word(epoch, kFlagA, aggregate));
    uint64_t excl = 0;
    int64_t hi = (int64_t)tile - 1;
    for (;;) {
        const int64_t idx = hi - tid;
        uint64_t s = kFlagP;                       // before tile 0: inclusive prefix 0
        if (idx >= 0) {
            do { s = ld_volatile(&states[idx]); } while ((uint32_t)(s >> 40) != epoch);
        }
        int mp = (s & kFlagP) ? tid : 0x7fffffff;  // nearest predecessor with a prefix
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) mp = min(mp, __shfl_xor_sync(kFull, mp, o));
        if (lane == 0) s_min[warp] = mp;
        __syncthreads();
        int nearest = s_min[0];
#pragma unroll
        for (int w = 1; w < NW; ++w) nearest = min(nearest, s_min[w]);
        const uint64_t wsum = warp_sum_u64(tid <= nearest ? (s & kValMask) : 0);
        if (lane == 0) s_sum[warp] = wsum;
        __syncthreads();
        uint64_t tot = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) tot += s_sum[w];
        excl += tot;
        __syncthreads();
        if (nearest != 0x7fffffff) break;
        hi -= NT;
    }
    if (tid == 0) st_volatile(&states[tile], state_word(epoch, kFlagP, excl + aggregate));
    return excl;
}

// Persistent-CTA tile ticket.  Every CTA draws until it gets a tile >= n_tiles;
// the CTA that draws last resets the counter for the next launch.
__device__ __forceinline__ uint64_t draw_tile(unsigned long long *ticket, uint64_t n_tiles,
                                              uint64_t *s_tile) {
    if (threadIdx.x == 0) {
        const uint64_t t = atomicAdd(ticket, 1ull);
        if (t == n_tiles + gridDim.x - 1) *ticket = 0ull;
        *s_tile = t;
    }
    __syncthreads();
    return *s_tile;
}

// ---------------------------------------------------------------------------
// ordered compaction over [0, n): pred = leaf digests differ (MODE 0) or a
// flag byte is set (MODE 1).  Output value = item index (a global chunk id).
// ---------------------------------------------------------------------------
constexpr int kCompactThreads = 256;
constexpr int kCompactRows = 4;                           // rows of 32 items per warp
constexpr int kCompactTile = kCompactThreads * kCompactRows;  // 1024 items
constexpr int kRowsPerLane = kCompactRows * 8 / 32;       // scan: row counts per lane

struct CompactParams {
    const uint4 *leaf_a;
    const uint4 *leaf_b;
    const uint8_t *flags;
    uint64_t n;
    uint64_t *out;
    uint64_t cap;
    uint64_t *count;          // device: total hits
    uint64_t *states;         // >= n_tiles entries (epoch-tagged, never cleared)
    unsigned long long *ticket;  // 0 on entry, 0 again on exit
    uint32_t epoch;
};

template <int MODE>
__global__ void __launch_bounds__(kCompactThreads) compact_kernel(const __grid_constant__ CompactParams p) {
    __shared__ uint32_t row_cnt[kCompactRows * 8];
    __shared__ uint32_t row_off[kCompactRows * 8];
    __shared__ uint64_t s_excl;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t n_tiles = (p.n + kCompactTile - 1) / kCompactTile;
    // static tile striding over a grid that is fully co-resident (host sizes it), so a
    // look-back only ever waits on tiles that resident CTAs are processing
    for (uint64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const uint64_t t0 = tile * kCompactTile;
        uint32_t bits[kCompactRows];
        bool hit[kCompactRows];
        // all loads first (one round trip per tile), then the ballots
        if (MODE == 0) {
            uint4 va[kCompactRows], vb[kCompactRows];
#pragma unroll
            for (int k = 0; k < kCompactRows; ++k) {
                const uint64_t i = t0 + (uint64_t)k * kCompactThreads + warp * 32 + lane;
                va[k] = vb[k] = make_uint4(0u, 0u, 0u, 0u);
                if (i < p.n) { va[k] = __ldcs(p.leaf_a + i); vb[k] = __ldcs(p.leaf_b + i); }
            }
#pragma unroll
            for (int k = 0; k < kCompactRows; ++k) hit[k] = digest_ne(va[k], vb[k]);
        } else {
#pragma unroll
            for (int k = 0; k < kCompactRows; ++k) {
                const uint64_t i = t0 + (uint64_t)k * kCompactThreads + warp * 32 + lane;
                hit[k] = i < p.n && p.flags[i] != 0;
            }
        }
#pragma unroll
        for (int k = 0; k < kCompactRows; ++k) {
            bits[k] = __ballot_sync(kFull, hit[k]);
            if (lane == 0) row_cnt[k * 8 + warp] = __popc(bits[k]);
        }
        __syncthreads();
        if (warp == 0) {
            // rows in item order: k major, warp minor -> flat index k*8+warp
            uint32_t v[kRowsPerLane], s = 0;
#pragma unroll
            for (int r = 0; r < kRowsPerLane; ++r) { v[r] = row_cnt[lane * kRowsPerLane + r]; s += v[r]; }
            uint32_t total;
            uint32_t ex = warp_excl_scan_u32(s, lane, total);
#pragma unroll
            for (int r = 0; r < kRowsPerLane; ++r) { row_off[lane * kRowsPerLane + r] = ex; ex += v[r]; }
            if (lane == 0) s_excl = total;
        }
        __syncthreads();
        const uint64_t total = s_excl;
        const uint64_t excl = cta_lookback<kCompactThreads>(p.states, tile, total, p.epoch);
        if (threadIdx.x == 0 && tile == n_tiles - 1) *p.count = excl + total;
        const uint32_t lt = (1u << lane) - 1u;
#pragma unroll
        for (int k = 0; k < kCompactRows; ++k) {
            if (bits[k] & (1u << lane)) {
                const uint64_t pos = excl + row_off[k * 8 + warp] + __popc(bits[k] & lt);
                if (pos < p.cap) p.out[pos] = t0 + (uint64_t)k * kCompactThreads + warp * 32 + lane;
            }
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// BFS steps for a start level above the leaves.
// Frontier entry: array (20 bits) | level (6 bits) | node (38 bits).
// ---------------------------------------------------------------------------
struct BfsParams {
    const uint4 *na;
    const uint4 *nb;
    const uint64_t *off;          // [level * n_arrays + a]
    const uint64_t *cnt;
    const uint64_t *chunk_base;   // [a] global chunk id of array a's leaf 0
    const uint64_t *sbegin;       // [a] prefix of start-level node counts (first step)
    const uint32_t *slevel;       // [a] start level of array a
    uint64_t n_start;             // total start-level nodes
    int n_arrays;
    uint8_t *flags;               // [total leaves] zeroed
};

__device__ __forceinline__ uint64_t pack_entry(uint64_t a, uint64_t l, uint64_t j) {
    return (a << 44) | (l << 38) | j;
}

__device__ __forceinline__ int find_u64(const uint64_t *v, int n, uint64_t x) {
    int lo = 0, hi = n - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (v[mid] <= x) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// Compare node (a,l,j); unequal leaves set their flag, unequal inner nodes
// push their children (warp-aggregated append).
__device__ __forceinline__ void bfs_visit(const BfsParams &p, bool valid, uint64_t a, uint64_t l,
                                          uint64_t j, uint64_t *out, unsigned long long *out_cnt,
                                          int lane) {
    uint32_t nchild = 0;
    uint64_t c0 = 0;
    if (valid) {
        const uint64_t o = p.off[l * p.n_arrays + a] + j;
        if (digest_ne(p.na[o], p.nb[o])) {
            if (l == 0) {
                p.flags[p.chunk_base[a] + j] = 1;
            } else {
                const uint64_t nd = p.cnt[(l - 1) * p.n_arrays + a];
                c0 = pack_entry(a, l - 1, 2 * j);
                nchild = (2 * j + 1 < nd) ? 2u : 1u;
            }
        }
    }
    uint32_t total;
    const uint32_t ex = warp_excl_scan_u32(nchild, lane, total);
    if (total == 0) return;
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(out_cnt, (unsigned long long)total);
    base = __shfl_sync(kFull, base, 0);
    for (uint32_t c = 0; c < nchild; ++c) out[base + ex + c] = c0 + c;
}

__global__ void bfs_first_kernel(BfsParams p, uint64_t *out, unsigned long long *out_cnt) {
    const int lane = threadIdx.x & 31;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t base = (uint64_t)blockIdx.x * blockDim.x; base < p.n_start; base += stride) {
        const uint64_t i = base + threadIdx.x;
        const bool valid = i < p.n_start;
        uint64_t a = 0, l = 0, j = 0;
        if (valid) {
            a = (uint64_t)find_u64(p.sbegin, p.n_arrays, i);
            l = p.slevel[a];
            j = i - p.sbegin[a];
        }
        bfs_visit(p, valid, a, l, j, out, out_cnt, lane);
    }
}

__global__ void bfs_step_kernel(BfsParams p, const uint64_t *in, const unsigned long long *in_cnt,
                                uint64_t *out, unsigned long long *out_cnt) {
    const int lane = threadIdx.x & 31;
    const uint64_t n = *in_cnt;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t base = (uint64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        const uint64_t i = base + threadIdx.x;
        const bool valid = i < n;
        uint64_t a = 0, l = 0, j = 0;
        if (valid) {
            const uint64_t e = in[i];
            a = e >> 44;
            l = (e >> 38) & 63;
            j = e & ((1ull << 38) - 1);
        }
        bfs_visit(p, valid, a, l, j, out, out_cnt, lane);
    }
}

// ---------------------------------------------------------------------------
// K4 verify: one warp per listed chunk, 8 chunks per tile.
// ---------------------------------------------------------------------------
constexpr int kVerifyWarps = 8;

struct VerifyArray {
    const uint8_t *a;
    const uint8_t *b;
    uint64_t n;            // elements
    uint64_t chunk_base;   // global chunk id of local chunk 0
    uint64_t elem_base;    // global element id of local element 0
};

constexpr int kVerifyInline = 16;   // array tables up to this size travel in the kernel params

struct VerifyParams {
    const VerifyArray *arrays;    // device table (n_arrays > kVerifyInline)
    const uint64_t *chunk_base;   // [a] copy of arrays[a].chunk_base for the search
    VerifyArray inl[kVerifyInline];
    uint64_t inl_base[kVerifyInline];
    int n_arrays;
    const uint64_t *chunks;
    const uint64_t *n_chunks_dev; // may be null -> n_chunks_host
    uint64_t n_chunks_host;
    uint64_t chunks_cap;
    uint32_t per;                 // elements per chunk
    double eps;
    uint64_t *out;
    uint64_t cap;
    uint64_t *count;
    uint64_t *states;
    unsigned long long *ticket;
    uint32_t epoch;
};

// 16-byte vector of elements starting at element e (e % VEC == 0); bits of
// |a-b| > eps for the elements < len.
template <int DT>
__device__ __forceinline__ uint32_t diff_bits(const uint8_t *pa, const uint8_t *pb, uint64_t e,
                                              uint64_t len, double eps) {
    constexpr int VEC = DT == 0 ? 4 : 2;
    uint32_t m = 0;
    if (e + VEC <= len) {
        const uint4 va = __ldg(reinterpret_cast<const uint4 *>(pa) + e / VEC);
        const uint4 vb = __ldg(reinterpret_cast<const uint4 *>(pb) + e / VEC);
        if (DT == 0) {
            m |= (fabs((double)__uint_as_float(va.x) - (double)__uint_as_float(vb.x)) > eps) ? 1u : 0u;
            m |= (fabs((double)__uint_as_float(va.y) - (double)__uint_as_float(vb.y)) > eps) ? 2u : 0u;
            m |= (fabs((double)__uint_as_float(va.z) - (double)__uint_as_float(vb.z)) > eps) ? 4u : 0u;
            m |= (fabs((double)__uint_as_float(va.w) - (double)__uint_as_float(vb.w)) > eps) ? 8u : 0u;
        } else {
            const double a0 = __hiloint2double((int)va.y, (int)va.x), b0 = __hiloint2double((int)vb.y, (int)vb.x);
            const double a1 = __hiloint2double((int)va.w, (int)va.z), b1 = __hiloint2double((int)vb.w, (int)vb.z);
            m |= (fabs(a0 - b0) > eps) ? 1u : 0u;
            m |= (fabs(a1 - b1) > eps) ? 2u : 0u;
        }
    } else {
        for (int v = 0; v < VEC; ++v) {
            if (e + v >= len) break;
            double x, y;
            if (DT == 0) {
                x = (double)reinterpret_cast<const float *>(pa)[e + v];
                y = (double)reinterpret_cast<const float *>(pb)[e + v];
            } else {
                x = reinterpret_cast<const double *>(pa)[e + v];
                y = reinterpret_cast<const double *>(pb)[e + v];
            }
            if (fabs(x - y) > eps) m |= 1u << v;
        }
    }
    return m;
}

template <int DT>
__global__ void __launch_bounds__(kVerifyWarps * 32) verify_kernel(const __grid_constant__ VerifyParams p) {
    constexpr int VEC = DT == 0 ? 4 : 2;
    constexpr int ESZ = DT == 0 ? 4 : 8;
    __shared__ uint32_t w_cnt[kVerifyWarps];
    __shared__ uint64_t s_excl;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint64_t n_chunks = p.n_chunks_dev ? *p.n_chunks_dev : p.n_chunks_host;
    if (n_chunks > p.chunks_cap) n_chunks = p.chunks_cap;
    const uint64_t n_tiles = (n_chunks + kVerifyWarps - 1) / kVerifyWarps;
    if (n_tiles == 0) {
        if (blockIdx.x == 0 && threadIdx.x == 0) *p.count = 0;
        return;
    }
    const uint32_t lt = (1u << lane) - 1u;
    for (uint64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const uint64_t q = tile * kVerifyWarps + warp;
        const bool have = q < n_chunks;
        const uint8_t *pa = nullptr, *pb = nullptr;
        uint64_t e_begin = 0, len = 0, gbase = 0;
        if (have) {
            const uint64_t g = p.chunks[q];
            const bool inl = p.n_arrays <= kVerifyInline;
            const int a = find_u64(inl ? p.inl_base : p.chunk_base, p.n_arrays, g);
            const VerifyArray A = inl ? p.inl[a] : p.arrays[a];
            const uint64_t c = g - A.chunk_base;
            e_begin = c * p.per;
            const uint64_t e_end = (e_begin + p.per) < A.n ? (e_begin + p.per) : A.n;
            len = e_end > e_begin ? e_end - e_begin : 0;
            pa = A.a + e_begin * ESZ;
            pb = A.b + e_begin * ESZ;
            gbase = A.elem_base + e_begin;
        }
        // pass 1: count; chunks of up to 64/VEC warp iterations keep their hit bits in
        // a register so pass 2 does not re-read the data
        uint32_t cnt = 0;
        uint64_t held = 0;
        constexpr int kStep = 32 * VEC;
        constexpr int kHeldIters = 64 / VEC;
        const bool hold = len <= (uint64_t)kHeldIters * kStep;
        {
            int it = 0;
#pragma unroll 4
            for (uint64_t e = (uint64_t)lane * VEC; e < len; e += kStep, ++it) {
                const uint32_t m = diff_bits<DT>(pa, pb, e, len, p.eps);
                cnt += __popc(m);
                if (it < kHeldIters) held |= (uint64_t)m << (it * VEC);
            }
        }
        cnt = (uint32_t)warp_sum_u64(cnt);
        if (lane == 0) w_cnt[warp] = cnt;
        __syncthreads();
        if (warp == 0) {
            const uint32_t v = lane < kVerifyWarps ? w_cnt[lane] : 0u;
            uint32_t total;
            const uint32_t ex = warp_excl_scan_u32(v, lane, total);
            __syncwarp();
            if (lane < kVerifyWarps) w_cnt[lane] = ex;
            if (lane == 0) s_excl = total;
        }
        __syncthreads();
        const uint64_t tile_total = s_excl;
        const uint64_t excl = cta_lookback<kVerifyWarps * 32>(p.states, tile, tile_total, p.epoch);
        if (threadIdx.x == 0 && tile == n_tiles - 1) *p.count = excl + tile_total;
        // pass 2: emit (only chunks with hits re-read their data)
        if (cnt) {
            uint64_t pos = excl + w_cnt[warp];
            int it = 0;
            for (uint64_t e0 = 0; e0 < len; e0 += kStep, ++it) {
                const uint64_t e = e0 + (uint64_t)lane * VEC;
                uint32_t m;
                if (hold) m = (uint32_t)(held >> (it * VEC)) & ((1u << VEC) - 1u);
                else m = e < len ? diff_bits<DT>(pa, pb, e, len, p.eps) : 0u;
                if (__ballot_sync(kFull, m != 0) == 0) continue;
                uint32_t total;
                const uint32_t ex = warp_excl_scan_u32(__popc(m), lane, total);
                uint32_t mm = m, k = 0;
                while (mm) {
                    const int bit = __ffs(mm) - 1;
                    mm &= mm - 1;
                    const uint64_t o = pos + ex + k++;
                    if (o < p.cap) p.out[o] = gbase + e + bit;
                }
                pos += total;
            }
        }
        (void)lt;
        __syncthreads();
    }
}

}  // namespace ckpt

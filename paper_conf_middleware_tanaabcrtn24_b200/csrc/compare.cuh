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
#include "mark.cuh"

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
// rows of 32 items per warp: 4 for digest pairs (MODE 0, 32 B per item), 16 for
// flag bytes (MODE 1: 4096-item tiles, so the look-back chain has 4x fewer
// links; with 1 KB tiles it set the compaction time, e.g. 78 us for 8.4 M flags)
template <int MODE> __host__ __device__ constexpr int compact_rows() { return MODE == 0 ? 4 : 16; }
template <int MODE> __host__ __device__ constexpr int compact_tile() { return kCompactThreads * compact_rows<MODE>(); }

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
    uint64_t base;            // added to every output index (a segment's global chunk id)
};

template <int MODE>
__global__ void __launch_bounds__(kCompactThreads) compact_kernel(const __grid_constant__ CompactParams p) {
    pdl_enter();
    constexpr int kCompactRows = compact_rows<MODE>();
    constexpr int kCompactTile = compact_tile<MODE>();
    constexpr int kRowsPerLane = kCompactRows * 8 / 32;       // scan: row counts per lane
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
                if (pos < p.cap) p.out[pos] = p.base + t0 + (uint64_t)k * kCompactThreads + warp * 32 + lane;
            }
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// Ordered chunk list of the fused pair path from K1's tile compaction
// (leaf.cuh, tile_compact): tile t's ids go to out[sum of tagg[0..t) ..].
// One pass, no look-back; CTA 0 also writes the total count.
// ---------------------------------------------------------------------------
struct TileGatherParams {
    const uint32_t *tagg;         // [n_tiles] flagged chunks per tile
    const uint64_t *tids;         // [n_tiles * tile_ids] tile-compacted chunk ids
    uint64_t n_tiles;
    uint64_t tile_ids;            // id slots per tile
    uint64_t *out;
    uint64_t cap;
    uint64_t *count;              // device: total flagged chunks
};

constexpr int kGatherThreads = 256;

__global__ void __launch_bounds__(kGatherThreads) tile_gather_kernel(const __grid_constant__ TileGatherParams p) {
    pdl_enter();
    __shared__ uint64_t s_red[kGatherThreads / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    auto block_sum = [&](uint64_t upto) -> uint64_t {   // sum of tagg[0..upto)
        uint64_t x = 0;
        for (uint64_t i = threadIdx.x; i < upto; i += kGatherThreads) x += p.tagg[i];
        x = warp_sum_u64(x);
        if (lane == 0) s_red[warp] = x;
        __syncthreads();
        uint64_t t = 0;
#pragma unroll
        for (int w = 0; w < kGatherThreads / 32; ++w) t += s_red[w];
        __syncthreads();
        return t;
    };
    if (blockIdx.x == 0) {
        const uint64_t total = block_sum(p.n_tiles);
        if (threadIdx.x == 0) *p.count = total;
    }
    for (uint64_t t = blockIdx.x; t < p.n_tiles; t += gridDim.x) {
        const uint64_t base = block_sum(t);
        const uint32_t n = p.tagg[t];
        const uint64_t *src = p.tids + t * p.tile_ids;
        for (uint32_t k = threadIdx.x; k < n; k += kGatherThreads)
            if (base + k < p.cap) p.out[base + k] = src[k];
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
    pdl_enter();
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
    pdl_enter();
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
// K4 verify, three kernels:
//   K4a verify_mark_kernel: warps walk groups of listed chunks (no inter-CTA
//       synchronisation), stream both runs once, and write each chunk's hit
//       count and hit bitmask (1 bit per element, element-contiguous 32-bit
//       words) to scratch.
//   K4b verify_scan_kernel: ordered exclusive scan of the counts (decoupled
//       look-back over 4 bytes per chunk) -> output offset per chunk.
//   K4c verify_emit_kernel: warps walk groups of chunks and write the element
//       ids of each chunk with hits from its bitmask (ascending, coalesced).
// The data pass never waits on a look-back chain.
// ---------------------------------------------------------------------------
constexpr int kVerifyWarps = 8;
constexpr int kVerifyThreads = kVerifyWarps * 32;

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
    uint32_t groups;              // mask words per lane per chunk
    double eps;
    uint32_t *cnt;                // [chunks_cap] hits per listed chunk (scratch)
    uint32_t *mask;               // [chunks_cap][groups][32] hit bits (scratch)
    uint64_t *off;                // [chunks_cap] output position of each chunk's first hit
    uint64_t *out;
    uint64_t cap;
    uint64_t *count;
    uint64_t *states;             // look-back state words (K4b)
    uint32_t epoch;
    // fused pair path: the chunk list is K1's tile compaction (leaf.cuh
    // tile_compact) read directly by K4a, which also writes it out (list_out,
    // n_chunks_out = the device count every later kernel reads as n_chunks_dev)
    const uint32_t *tagg;         // [n_tiles] flagged chunks per tile, or null
    const uint64_t *tids;         // [n_tiles * tile_ids]
    uint32_t n_tiles;
    uint32_t tile_ids;
    uint64_t *list_out;
    uint64_t *n_chunks_out;
};

constexpr int kVerifyMaxTiles = 4096;   // tile prefix table of K4a in shared memory

__device__ __forceinline__ uint64_t verify_n_chunks(const VerifyParams &p) {
    const uint64_t n = p.n_chunks_dev ? *p.n_chunks_dev : p.n_chunks_host;
    return n < p.chunks_cap ? n : p.chunks_cap;
}

// Locate listed chunk q: data pointers at its first element, its length and
// the global id of its first element.
__device__ __forceinline__ void verify_locate_g(const VerifyParams &p, uint64_t g, int esz,
                                                const uint8_t *&pa, const uint8_t *&pb,
                                                uint64_t &len, uint64_t &gbase) {
    const bool inl = p.n_arrays <= kVerifyInline;
    const int a = find_u64(inl ? p.inl_base : p.chunk_base, p.n_arrays, g);
    const VerifyArray A = inl ? p.inl[a] : p.arrays[a];
    const uint64_t e_begin = (g - A.chunk_base) * p.per;
    const uint64_t e_end = (e_begin + p.per) < A.n ? (e_begin + p.per) : A.n;
    len = e_end > e_begin ? e_end - e_begin : 0;
    pa = A.a + e_begin * esz;
    pb = A.b + e_begin * esz;
    gbase = A.elem_base + e_begin;
}

__device__ __forceinline__ void verify_locate(const VerifyParams &p, uint64_t q, int esz,
                                              const uint8_t *&pa, const uint8_t *&pb,
                                              uint64_t &len, uint64_t &gbase) {
    verify_locate_g(p, p.chunks[q], esz, pa, pb, len, gbase);
}

// Tile mode: exclusive prefix of the tile counts into s_tpre[0..n_tiles]
// (s_tpre[n_tiles] = total).  Called by all threads of the CTA.
__device__ __forceinline__ void tile_prefix(const VerifyParams &p, uint32_t *s_tpre) {
    __shared__ uint32_t s_w[kVerifyWarps];
    constexpr int kPer = kVerifyMaxTiles / kVerifyThreads;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t nt = p.n_tiles;
    const uint32_t t0 = threadIdx.x * kPer;
    uint32_t v[kPer], sum = 0;
#pragma unroll
    for (int k = 0; k < kPer; ++k) {
        v[k] = t0 + k < nt ? __ldcg(p.tagg + t0 + k) : 0u;
        sum += v[k];
    }
    uint32_t wt;
    uint32_t ex = warp_excl_scan_u32(sum, lane, wt);
    if (lane == 0) s_w[warp] = wt;
    __syncthreads();
#pragma unroll
    for (int w = 0; w < kVerifyWarps; ++w) ex += w < warp ? s_w[w] : 0u;
#pragma unroll
    for (int k = 0; k < kPer; ++k) {
        if (t0 + k <= nt) s_tpre[t0 + k] = ex;
        ex += v[k];
    }
    if (threadIdx.x == kVerifyThreads - 1 && nt == kVerifyMaxTiles) s_tpre[nt] = ex;
    __syncthreads();
}

// Tile mode: chunk id of list position q (q < total).
__device__ __forceinline__ uint64_t tile_chunk(const VerifyParams &p, const uint32_t *s_tpre, uint64_t q) {
    uint32_t lo = 0, hi = p.n_tiles - 1;               // last tile with s_tpre[t] <= q
    while (lo < hi) {
        const uint32_t mid = (lo + hi + 1) >> 1;
        if (s_tpre[mid] <= q) lo = mid; else hi = mid - 1;
    }
    return __ldcg(reinterpret_cast<const unsigned long long *>(p.tids) + (uint64_t)lo * p.tile_ids +
                  (q - s_tpre[lo]));
}

// Chunks per warp group: the largest power of two <= 32 that still gives
// every warp of the grid a group.  The lanes of a warp locate the group's
// chunks in parallel (one binary search each) and the warp then walks them, so
// the dependent loads of the search are paid once per group, not per chunk.
__device__ __forceinline__ uint32_t verify_group(uint64_t n_chunks, uint64_t n_warps) {
    uint32_t g = 32;
    while (g > 1 && (uint64_t)g * n_warps > n_chunks) g >>= 1;
    return g;
}

struct ChunkLoc {
    const uint8_t *pa, *pb;
    uint64_t len, gbase;
};

__device__ __forceinline__ ChunkLoc shfl_loc(const ChunkLoc &l, int src) {
    ChunkLoc o;
    o.pa = (const uint8_t *)__shfl_sync(kFull, (unsigned long long)l.pa, src);
    o.pb = (const uint8_t *)__shfl_sync(kFull, (unsigned long long)l.pb, src);
    o.len = __shfl_sync(kFull, l.len, src);
    o.gbase = __shfl_sync(kFull, l.gbase, src);
    return o;
}

template <int DT>
__global__ void __launch_bounds__(kVerifyThreads) verify_mark_kernel(const __grid_constant__ VerifyParams p) {
    pdl_enter();
    constexpr int ESZ = DT == 0 ? 4 : 8;
    __shared__ uint32_t s_tpre[kVerifyMaxTiles + 1];
    const int lane = threadIdx.x & 31;
    uint64_t n_chunks;
    if (p.tagg) {
        tile_prefix(p, s_tpre);
        const uint64_t total = s_tpre[p.n_tiles];
        if (blockIdx.x == 0 && threadIdx.x == 0) *p.n_chunks_out = total;
        n_chunks = total < p.chunks_cap ? total : p.chunks_cap;
    } else {
        n_chunks = verify_n_chunks(p);
    }
    const uint64_t n_warps = (uint64_t)gridDim.x * kVerifyWarps;
    const uint32_t G = verify_group(n_chunks, n_warps);
    for (uint64_t q0 = ((uint64_t)blockIdx.x * kVerifyWarps + (threadIdx.x >> 5)) * G; q0 < n_chunks;
         q0 += n_warps * G) {
      ChunkLoc mine{nullptr, nullptr, 0, 0};
      if (lane < (int)G && q0 + lane < n_chunks) {
          if (p.tagg) {
              const uint64_t g = tile_chunk(p, s_tpre, q0 + lane);
              p.list_out[q0 + lane] = g;
              verify_locate_g(p, g, ESZ, mine.pa, mine.pb, mine.len, mine.gbase);
          } else {
              verify_locate(p, q0 + lane, ESZ, mine.pa, mine.pb, mine.len, mine.gbase);
          }
      }
      const uint32_t nq = (n_chunks - q0) < G ? (uint32_t)(n_chunks - q0) : G;
      for (uint32_t j = 0; j < nq; ++j) {
        const uint64_t q = q0 + j;
        const ChunkLoc L = shfl_loc(mine, j);
        const uint8_t *pa = L.pa, *pb = L.pb;
        const uint64_t len = L.len;
        const uint32_t cnt = mark_chunk<DT>(pa, pb, len, p.eps, p.mask + q * p.groups * 32, lane);
        if (lane == 0) p.cnt[q] = cnt;
      }
    }
}

// K4b: exclusive scan of the per-chunk hit counts (kVerifyScanItems chunks per
// thread, decoupled look-back across tiles) -> p.off[q]; the last tile writes
// the total to *p.count.
constexpr int kVerifyScanItems = 4;
constexpr int kVerifyScanTile = kVerifyThreads * kVerifyScanItems;

__global__ void __launch_bounds__(kVerifyThreads) verify_scan_kernel(const __grid_constant__ VerifyParams p) {
    pdl_enter();
    __shared__ uint64_t w_tot[kVerifyWarps];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t n_chunks = verify_n_chunks(p);
    const uint64_t n_tiles = (n_chunks + kVerifyScanTile - 1) / kVerifyScanTile;
    if (n_tiles == 0) {
        if (blockIdx.x == 0 && threadIdx.x == 0) *p.count = 0;
        return;
    }
    for (uint64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const uint64_t q0 = tile * kVerifyScanTile + (uint64_t)threadIdx.x * kVerifyScanItems;
        uint32_t c[kVerifyScanItems];
        uint64_t sum = 0;
#pragma unroll
        for (int k = 0; k < kVerifyScanItems; ++k) {
            c[k] = q0 + k < n_chunks ? p.cnt[q0 + k] : 0u;
            sum += c[k];
        }
        uint64_t x = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint64_t y = __shfl_up_sync(kFull, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) w_tot[warp] = x;
        __syncthreads();
        uint64_t before = 0, total = 0;
#pragma unroll
        for (int w = 0; w < kVerifyWarps; ++w) {
            const uint64_t v = w_tot[w];
            if (w < warp) before += v;
            total += v;
        }
        const uint64_t excl = cta_lookback<kVerifyThreads>(p.states, tile, total, p.epoch);
        if (threadIdx.x == 0 && tile == n_tiles - 1) *p.count = excl + total;
        uint64_t pos = excl + before + x - sum;
#pragma unroll
        for (int k = 0; k < kVerifyScanItems; ++k) {
            if (q0 + k < n_chunks) p.off[q0 + k] = pos;
            pos += c[k];
        }
        __syncthreads();
    }
}

// Write the hits of one group of 32 mask words (1024 elements from e_base,
// word l in lane l) to out[pos..).  The hit offsets are first compacted into
// the warp's shared-memory slot (lane l after the hits of lanes < l), then
// written out with each store instruction covering 32 consecutive output slots.
// Returns the count.
__device__ __forceinline__ uint32_t emit_words(uint32_t word, uint64_t e_base, uint64_t pos,
                                               uint64_t *out, uint64_t cap, int lane,
                                               uint16_t *s_off) {
    if (__ballot_sync(kFull, word != 0) == 0) return 0;
    uint32_t tot;
    uint32_t o = warp_excl_scan_u32(__popc(word), lane, tot);
    for (uint32_t mm = word; mm; mm &= mm - 1, ++o) s_off[o] = (uint16_t)(lane * 32 + __ffs(mm) - 1);
    __syncwarp();
    for (uint32_t k = lane; k < tot; k += 32)
        if (pos + k < cap) out[pos + k] = e_base + s_off[k];
    __syncwarp();
    return tot;
}

// K4c: warps walk groups of listed chunks; the lanes load the group's counts,
// offsets and locations in parallel.  Sparse chunks (<= kEmitSparse hits) are
// emitted one per lane (the lane reads the chunk's mask words with 16-byte
// loads and writes its ids in order); dense chunks are emitted by the whole
// warp, one 32-word group at a time, with coalesced stores.
constexpr uint32_t kEmitSparse = 48;

template <int DT>
__global__ void __launch_bounds__(kVerifyThreads) verify_emit_kernel(const __grid_constant__ VerifyParams p) {
    pdl_enter();
    constexpr int ESZ = DT == 0 ? 4 : 8;
    __shared__ uint16_t s_off_all[kVerifyWarps][1024];
    const int lane = threadIdx.x & 31;
    uint16_t *s_off = s_off_all[threadIdx.x >> 5];
    const uint64_t n_chunks = verify_n_chunks(p);
    const uint64_t n_warps = (uint64_t)gridDim.x * kVerifyWarps;
    const uint32_t G = verify_group(n_chunks, n_warps);
    const uint32_t n_words = p.groups * 32;
    for (uint64_t q0 = ((uint64_t)blockIdx.x * kVerifyWarps + (threadIdx.x >> 5)) * G; q0 < n_chunks;
         q0 += n_warps * G) {
      uint64_t my_off = 0, my_gb = 0, my_key = 0;
      uint32_t c = 0, my_groups = 0;
      if (lane < (int)G && q0 + lane < n_chunks) {
          my_key = q0 + lane;
          c = p.cnt[my_key];
          if (c) {
              const uint8_t *pa, *pb;
              uint64_t len;
              my_off = p.off[q0 + lane];
              verify_locate(p, q0 + lane, ESZ, pa, pb, len, my_gb);
              // mark_chunk wrote ceil(len/1024) groups; the rest of the chunk's slot holds
              // stale words (a short last chunk of an array) and must not be read
              my_groups = (uint32_t)((len + 1023) / 1024);
          }
      }
      // sparse chunks: one lane each
      if (c && c <= kEmitSparse) {
          const uint4 *mw = reinterpret_cast<const uint4 *>(p.mask + my_key * n_words);
          uint64_t o = my_off;
#pragma unroll 1
          for (uint32_t w4 = 0; w4 < my_groups * 8u; ++w4) {
              const uint4 v = __ldcs(mw + w4);
              const uint32_t wv[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
              for (int k = 0; k < 4; ++k) {
                  const uint64_t e = my_gb + (uint64_t)(w4 * 4 + k) * 32;
                  for (uint32_t mm = wv[k]; mm; mm &= mm - 1, ++o)
                      if (o < p.cap) p.out[o] = e + (__ffs(mm) - 1);
              }
          }
      }
      // dense chunks: the whole warp
#pragma unroll 1
      for (uint32_t todo = __ballot_sync(kFull, c > kEmitSparse); todo; todo &= todo - 1) {
        const int j = __ffs(todo) - 1;
        const uint64_t gbase = __shfl_sync(kFull, my_gb, j);
        uint64_t pos = __shfl_sync(kFull, my_off, j);
        const uint32_t groups = __shfl_sync(kFull, my_groups, j);
        const uint32_t *mq = p.mask + __shfl_sync(kFull, my_key, j) * n_words + lane;
#pragma unroll 1
        for (uint32_t g = 0; g < groups; ++g)
            pos += emit_words(__ldcs(mq + g * 32), gbase + (uint64_t)g * 1024, pos, p.out, p.cap, lane,
                              s_off);
      }
    }
}

}  // namespace ckpt

// levels.cuh -- K2: interior Merkle levels, several trees, one launch.
//
// Paper: Alg. 1 lines 13-20 -- "for all node in level do in
// parallel: Tree(node) <- hash({left, right})", levels bottom-up; flattened
// array storage.  Reading R13: n_{l+1} = ceil(n_l/2), an odd last
// node is promoted unchanged, so any aligned group of 2^G nodes of a level is
// an exact subtree.
//
// Phase 1 (every CTA, one per aligned group of 2048 nodes of level ls of one
//   array): passes of two levels through shared memory -- in each pass the
//   first ceil(cnt/4) of the 512 threads take 4 consecutive nodes and hash them
//   two levels up (2 independent hashes, then 1), writing both levels.
// Phase 2 (last CTA of each tree, acq_rel ticket): loads the remaining level
//   of every array into shared memory, builds all upper levels there, then
//   the top tree over the array roots (R15).  Levels that do not fit in
//   shared memory are walked through L2.
#pragma once
#include <cstdint>

#include "hash.cuh"
#include "mm32.cuh"

namespace ckpt {

constexpr int kLevelThreads = 512;
constexpr int kLog = 11;
constexpr int kGroup = 1 << kLog;            // nodes of level ls per CTA (512 threads x 4)
constexpr int kLevelSmemNodes = 1536;        // phase-2 shared memory in nodes (24 KiB)
constexpr int kLevelSmem = kLevelSmemNodes * 16;
constexpr int kMaxLevelTrees = 4;

constexpr int kLevelInlineWords = 512;   // 4 KiB of tree metadata in the kernel params
constexpr int kLevelTabWords = 512;      // phase 2: level tables staged in shared memory

// Per-tree launch record.  The metadata tables live in one blob (layout below)
// that is either inline in the kernel parameters (small trees: no H2D copy;
// the tree's first CTA then writes it to `meta` for later BFS use) or already
// in device memory at `meta`.
struct LevelParams {
    uint4 *nodes;                 // whole tree storage
    uint8_t *meta;                // device metadata blob
    int inl;                      // word offset of the blob in LevelBatch::blob, or -1
    uint32_t meta_words;
    // byte offsets in the blob:
    uint32_t o_off;               // u64 [level * n_arrays + a]: node index of array a's level
    uint32_t o_cnt;               // u64 [level * n_arrays + a]: node count (0 above the root)
    uint32_t o_lb;                // u64 [level]: node index of level (all arrays)
    uint32_t o_lt;                // u64 [level]: nodes in level (all arrays)
    uint32_t o_h;                 // u32 [a]: number of levels of array a
    uint32_t o_g;                 // u64 [a]: first group of array a
    uint64_t top_off;             // node index of the top tree's level 0
    unsigned int *ticket;         // zero on entry, reset to zero by the last CTA
    int n_arrays;
    int n_levels;                 // max height over arrays
    int ls;                       // start level of this launch
    unsigned int n_groups;        // CTAs of this tree
};

struct LevelBatch {
    LevelParams t[kMaxLevelTrees];
    unsigned int cta_begin[kMaxLevelTrees + 1];
    int n;
    uint64_t blob[kLevelInlineWords];
};

// Resolved view of one tree's tables.
struct LvView {
    uint4 *nodes;
    const uint64_t *off, *cnt, *gbegin, *level_base, *level_total;
    const uint32_t *height;
    uint64_t top_off;
    unsigned int *ticket;
    int n_arrays, n_levels, ls;
    unsigned int n_groups;
};

__device__ __forceinline__ int find_le(const uint64_t *v, int n, uint64_t x) {
    int lo = 0, hi = n - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (v[mid] <= x) lo = mid; else hi = mid - 1;
    }
    return lo;
}

__device__ __forceinline__ uint4 shfl_down4(uint4 v, int d) {
    return make_uint4(__shfl_down_sync(0xffffffffu, v.x, d), __shfl_down_sync(0xffffffffu, v.y, d),
                      __shfl_down_sync(0xffffffffu, v.z, d), __shfl_down_sync(0xffffffffu, v.w, d));
}

// Levels k0..k1 (relative to the warp's level-(k0-1) nodes held one per lane
// in `v`, `m` of them valid) with shuffles.  Node j of relative level k lives
// in lane j << (k - k0 + 1) ... written to global through `write(k, j, v)`.
template <class W>
__device__ __forceinline__ uint4 warp_levels(uint4 v, int m, int k0, int k1, int lane, W write) {
    for (int k = k0, step = 1; k <= k1; ++k, step <<= 1) {
        const uint4 r = shfl_down4(v, step);
        const int mk = (m + 1) >> 1;
        const int j = lane / (2 * step);
        if ((lane & (2 * step - 1)) == 0 && j < mk) {
            if (2 * j + 1 < m) v = hash_children32(v, r);
            write(k, j, v);
        }
        m = mk;
    }
    return v;
}

// One level over all arrays, children read from `src` (indexable by node
// index - src_base) and parents written to global and, if dst != null, to dst.
__device__ __forceinline__ void build_level(const LvView &p, int l, const uint4 *src,
                                            uint64_t src_base, uint4 *dst, bool from_global) {
    const int na = p.n_arrays;
    const uint64_t total = p.level_total[l];
    const uint64_t base = p.level_base[l];
    const uint64_t *off_l = p.off + (uint64_t)l * na;
    const uint64_t *off_d = p.off + (uint64_t)(l - 1) * na;
    const uint64_t *cnt_d = p.cnt + (uint64_t)(l - 1) * na;
    for (uint64_t i = threadIdx.x; i < total; i += blockDim.x) {
        const int a = find_le(off_l, na, base + i);
        const uint64_t j = base + i - off_l[a];
        const uint64_t c = off_d[a] + 2 * j - src_base;
        uint4 v = from_global ? __ldcg(src + c) : src[c];
        if (2 * j + 1 < cnt_d[a]) v = hash_children32(v, from_global ? __ldcg(src + c + 1) : src[c + 1]);
        p.nodes[base + i] = v;
        if (dst) dst[i] = v;
    }
}


__global__ void __launch_bounds__(kLevelThreads, 3) levels_kernel(const __grid_constant__ LevelBatch pb) {
    pdl_enter();
    extern __shared__ __align__(16) uint4 sm[];
    __shared__ unsigned int s_ticket;
    const int tid = threadIdx.x;
    int ti = 0;
    while (ti + 1 < pb.n && blockIdx.x >= pb.cta_begin[ti + 1]) ++ti;
    const LevelParams &lp = pb.t[ti];
    const uint8_t *mb = lp.inl >= 0 ? reinterpret_cast<const uint8_t *>(pb.blob + lp.inl) : lp.meta;
    LvView p;
    p.nodes = lp.nodes;
    p.off = reinterpret_cast<const uint64_t *>(mb + lp.o_off);
    p.cnt = reinterpret_cast<const uint64_t *>(mb + lp.o_cnt);
    p.level_base = reinterpret_cast<const uint64_t *>(mb + lp.o_lb);
    p.level_total = reinterpret_cast<const uint64_t *>(mb + lp.o_lt);
    p.height = reinterpret_cast<const uint32_t *>(mb + lp.o_h);
    p.gbegin = reinterpret_cast<const uint64_t *>(mb + lp.o_g);
    p.top_off = lp.top_off;
    p.ticket = lp.ticket;
    p.n_arrays = lp.n_arrays;
    p.n_levels = lp.n_levels;
    p.ls = lp.ls;
    p.n_groups = lp.n_groups;
    const int na = p.n_arrays;
    if (lp.inl >= 0 && blockIdx.x == pb.cta_begin[ti]) {
        // publish the inline tables to device memory for later BFS launches
        uint64_t *dst = reinterpret_cast<uint64_t *>(lp.meta);
        for (uint32_t w = tid; w < lp.meta_words; w += kLevelThreads) dst[w] = pb.blob[lp.inl + w];
    }
    // ------------------------------ phase 1 ------------------------------
    {
        // Passes of two levels through shared memory: in pass r/2 the first
        // ceil(cnt/4) threads each take 4 consecutive level-r nodes of the
        // group (cnt valid), hash them up to one level-(r+2) node (2 + 1
        // hashes, the first two independent) and store it for the next pass.
        // Every pass but the last few keeps whole warps busy, so the CTA's
        // 2047 hashes cost ~2047/32 warp-hashes instead of a lane-halving
        // shuffle tree, and 16 warps per CTA hide the hash latency.
        const uint64_t gid = blockIdx.x - pb.cta_begin[ti];
        const int a = find_le(p.gbegin, na, gid);
        const uint64_t g = gid - p.gbegin[a];
        const uint64_t n0 = p.cnt[(uint64_t)p.ls * na + a];
        const uint64_t start = g * kGroup;
        const int m0 = (int)((n0 - start) < (uint64_t)kGroup ? (n0 - start) : (uint64_t)kGroup);
        const int h = (int)p.height[a];
        const uint4 *src = p.nodes + p.off[(uint64_t)p.ls * na + a] + start;
        // the group's first node on each of its levels, formed once (threads 0..kLog in
        // parallel): the level tables are not re-read on the dependent path of the passes
        __shared__ uint4 *s_lvb[kLog + 1];
        if (tid <= kLog && p.ls + tid < h)
            s_lvb[tid] = p.nodes + p.off[(uint64_t)(p.ls + tid) * na + a] + (start >> tid);
        __syncthreads();
        auto write = [&](int k, uint64_t j, uint4 v) {
            if (p.ls + k < h) s_lvb[k][j] = v;
        };
        uint4 *buf[2] = {sm, sm + kLevelThreads};       // ping-pong: 512 + 128 nodes
        int cnt = m0;
        if (m0 == kGroup) {
            // full group (the common case): every level up to kLog exists in the array's
            // tree and every thread that works has 4 (or 2) valid nodes -- no predicates,
            // level base pointers formed once per pass
            for (int r = 0; r < kLog; r += 2) {
                const bool two = r + 2 <= kLog;
                const int need = two ? (kGroup >> r) >> 2 : (kGroup >> r) >> 1;
                const uint4 *in = buf[(r >> 1) & 1];
                uint4 *out = buf[((r >> 1) + 1) & 1];
                if (tid < need) {
                    uint4 *l1 = s_lvb[r + 1];
                    if (two) {
                        uint4 *l2 = s_lvb[r + 2];
                        uint4 x0, x1, x2, x3;
                        if (r == 0) {
                            x0 = __ldg(src + 4 * tid); x1 = __ldg(src + 4 * tid + 1);
                            x2 = __ldg(src + 4 * tid + 2); x3 = __ldg(src + 4 * tid + 3);
                        } else {
                            x0 = in[4 * tid]; x1 = in[4 * tid + 1]; x2 = in[4 * tid + 2]; x3 = in[4 * tid + 3];
                        }
                        const uint4 y0 = hash_children32(x0, x1);
                        const uint4 y1 = hash_children32(x2, x3);
                        l1[2 * tid] = y0;
                        l1[2 * tid + 1] = y1;
                        const uint4 z = hash_children32(y0, y1);
                        l2[tid] = z;
                        out[tid] = z;
                    } else {
                        const uint4 y0 = hash_children32(in[2 * tid], in[2 * tid + 1]);
                        l1[tid] = y0;
                        out[tid] = y0;
                    }
                }
                __syncthreads();
            }
            cnt = 1;
        }
        for (int r = 0; r < kLog && m0 != kGroup; r += 2) {
            const bool two = r + 2 <= kLog;
            const int need = two ? (cnt + 3) >> 2 : (cnt + 1) >> 1;
            const uint4 *in = buf[(r >> 1) & 1];
            uint4 *out = buf[((r >> 1) + 1) & 1];
            if (tid < need) {
                const int per = two ? 4 : 2;
                int mt = cnt - per * tid;
                mt = mt > per ? per : mt;
                uint4 x[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    x[j] = make_uint4(0u, 0u, 0u, 0u);
                    if (j < mt) x[j] = r == 0 ? __ldg(src + per * tid + j) : in[per * tid + j];
                }
                const uint4 y0 = mt >= 2 ? hash_children32(x[0], x[1]) : x[0];
                write(r + 1, (uint64_t)(per / 2) * tid, y0);
                if (two) {
                    uint4 y1 = make_uint4(0u, 0u, 0u, 0u);
                    if (mt >= 3) {
                        y1 = mt == 4 ? hash_children32(x[2], x[3]) : x[2];
                        write(r + 1, (uint64_t)2 * tid + 1, y1);
                    }
                    const uint4 z = mt >= 3 ? hash_children32(y0, y1) : y0;
                    write(r + 2, (uint64_t)tid, z);
                    out[tid] = z;
                } else {
                    out[tid] = y0;
                }
            }
            cnt = need;
            __syncthreads();
        }
    }
    // ------------------------------ phase 2 ------------------------------
    // Last-CTA hand-off without sequentially consistent fences (MEMBAR.SC.GPU
    // costs microseconds): the barrier orders every thread's node stores before
    // thread 0's acq_rel atomic, whose release is cumulative over them; in the
    // last CTA the same atomic acquires every other CTA's release, and the
    // next barrier extends that to all of its threads.
    __syncthreads();
    if (tid == 0) {
        unsigned int t;
        asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(t) : "l"(p.ticket) : "memory");
        s_ticket = t;
    }
    __syncthreads();
    if (s_ticket != p.n_groups - 1) return;
    {
        // the last CTA walks the level tables for every node it builds: stage them in shared
        // memory when they fit (a few KB for a handful of arrays)
        __shared__ uint64_t s_tab[kLevelTabWords];
        const uint32_t nl = (uint32_t)p.n_levels;
        const uint32_t nt = nl * (uint32_t)na;
        if (2 * nt + 2 * (nl + 1) <= (uint32_t)kLevelTabWords) {
            for (uint32_t i = tid; i < nt; i += kLevelThreads) {
                s_tab[i] = p.off[i];
                s_tab[nt + i] = p.cnt[i];
            }
            for (uint32_t i = tid; i <= nl; i += kLevelThreads) {
                s_tab[2 * nt + i] = p.level_base[i];
                s_tab[2 * nt + nl + 1 + i] = p.level_total[i];
            }
            __syncthreads();
            p.off = s_tab;
            p.cnt = s_tab + nt;
            p.level_base = s_tab + 2 * nt;
            p.level_total = s_tab + 2 * nt + nl + 1;
        }
    }
    int F = p.ls + kLog;                       // highest level phase 1 completed
    if (F > p.n_levels - 1) F = p.n_levels - 1;
    if (F + 1 <= p.n_levels - 1) {
        const uint64_t nF = p.level_total[F];
        const uint64_t nF1 = p.level_total[F + 1];
        if (nF + nF1 <= (uint64_t)kLevelSmemNodes) {
            // whole remainder in shared memory: ping-pong between two regions
            uint4 *cur = sm, *nxt = sm + nF;
            for (uint64_t i = tid; i < nF; i += kLevelThreads) cur[i] = __ldcg(p.nodes + p.level_base[F] + i);
            __syncthreads();
            for (int l = F + 1; l < p.n_levels; ++l) {
                build_level(p, l, cur, p.level_base[l - 1], nxt, false);
                __syncthreads();
                uint4 *t = cur;
                cur = nxt;
                nxt = t;
            }
        } else {
            for (int l = F + 1; l < p.n_levels; ++l) {
                build_level(p, l, p.nodes + p.level_base[l - 1], p.level_base[l - 1], nullptr, true);
                __syncthreads();
            }
        }
    }
    __syncthreads();
    // top tree: level 0 = array roots in array order (R15).  Up to 2 * kLevelSmemNodes / 3
    // roots it is built in shared memory (one L2 round trip for the roots, then only
    // stores); larger tops through L2.
    if ((uint64_t)na + ((uint64_t)na + 1) / 2 <= (uint64_t)kLevelSmemNodes) {
        uint4 *cur = sm, *nxt = sm + na;
        for (int a = tid; a < na; a += kLevelThreads) {
            const int h = (int)p.height[a];
            const uint4 v = __ldcg(p.nodes + p.off[(uint64_t)(h - 1) * na + a]);
            p.nodes[p.top_off + a] = v;
            cur[a] = v;
        }
        __syncthreads();
        uint64_t n = (uint64_t)na, at = p.top_off;
        while (n > 1) {
            const uint64_t up = (n + 1) >> 1;
            for (uint64_t j = tid; j < up; j += kLevelThreads) {
                uint4 x = cur[2 * j];
                if (2 * j + 1 < n) x = hash_children32(x, cur[2 * j + 1]);
                p.nodes[at + n + j] = x;
                nxt[j] = x;
            }
            __syncthreads();
            uint4 *t = cur;
            cur = nxt;
            nxt = t;
            at += n;
            n = up;
        }
        if (tid == 0) *p.ticket = 0u;
        return;
    }
    for (int a = tid; a < na; a += kLevelThreads) {
        const int h = (int)p.height[a];
        p.nodes[p.top_off + a] = __ldcg(p.nodes + p.off[(uint64_t)(h - 1) * na + a]);
    }
    __syncthreads();
    uint64_t n = (uint64_t)na, cur = p.top_off;
    while (n > 1) {
        const uint64_t up = (n + 1) >> 1;
        for (uint64_t j = tid; j < up; j += kLevelThreads) {
            uint4 x = __ldcg(p.nodes + cur + 2 * j);
            if (2 * j + 1 < n) x = hash_children32(x, __ldcg(p.nodes + cur + 2 * j + 1));
            p.nodes[cur + n + j] = x;
        }
        __syncthreads();
        cur += n;
        n = up;
    }
    if (tid == 0) *p.ticket = 0u;
}

}  // namespace ckpt

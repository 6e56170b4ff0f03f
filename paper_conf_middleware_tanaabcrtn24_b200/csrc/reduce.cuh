// reduce.cuh -- interior levels for the finish kernel (finish.cuh).
//
// Alg. 1 lines 13-20, reading R13/R14: node j of level l+1 is
// Murmur3F(node 2j || node 2j+1, 32 B, seed 0), or node 2j promoted when it has no right
// sibling.  Any aligned block of 2^k nodes of a level is an exact subtree, so a CTA can reduce
// a block of up to 512 nodes to its root on its own.  The levels kernel (levels.cuh) does it in
// passes of two levels through shared memory, which keeps lanes busy when there are many
// groups, and hands everything above the groups to one CTA; here a block is reduced the same
// way (passes of two levels, whole warps busy) down to 32 nodes, warp 0 finishes with
// shuffles, and the levels above the blocks are built by the last block of each array (then
// of each tree), in parallel over arrays.  Every node produced is stored at its place.
#pragma once
#include <cstdint>

#include "levels.cuh"
#include "mm32.cuh"

namespace ckpt {

constexpr int kRedThreads = 128;                 // the finish kernel's CTA
constexpr int kRedBlockLog = 9;                  // nodes per block: 2^9 = 128 threads x 4

// A tree's addressing: array levels from the metadata tables, the top tree over the array
// roots (array index na) after them, level-ordered.
struct TreeRef {
    uint4 *nodes;
    const uint64_t *off, *cnt;    // [level * na + a]
    const uint32_t *height;       // [a]
    uint64_t top_off;
    int na;

    __device__ __forceinline__ int levels(int aa) const {
        if (aa < na) return (int)height[aa];
        uint64_t n = (uint64_t)na;
        int h = 1;
        while (n > 1) { n = (n + 1) >> 1; ++h; }
        return h;
    }
    __device__ __forceinline__ uint64_t count(int aa, int k) const {
        if (aa < na) return cnt[(uint64_t)k * na + aa];
        return ((uint64_t)na + (1ull << k) - 1) >> k;
    }
    __device__ __forceinline__ uint4 *at(int aa, int k, uint64_t j) const {
        if (aa < na) return nodes + off[(uint64_t)k * na + aa] + j;
        uint64_t o = top_off, n = (uint64_t)na;
        for (int q = 0; q < k; ++q) { o += n; n = (n + 1) >> 1; }
        return nodes + o + j;
    }
};

// Levels l0+1 .. l0+kmax (kmax <= 9) of the block of m <= 512 level-l0 nodes of array aa
// starting at node s0 (s0 a multiple of 2^9).  Passes of two levels: the first ceil(c/4)
// threads each take 4 consecutive nodes (2 independent hashes, then 1) -- whole warps busy --
// until at most 32 nodes remain, which warp 0 takes the rest of the way with shuffles.
// Called by all kRedThreads threads; sm: 2 x kRedThreads nodes of shared memory.
__device__ __noinline__ void reduce_block(const TreeRef &T, int aa, int l0, uint64_t s0, uint32_t m,
                                          int kmax, uint4 *sm) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    uint4 *buf[2] = {sm, sm + kRedThreads};
    // the block's start node on each level l0 .. l0+kmax, once (the tables live in the kernel
    // parameters or global memory; every node store below addresses through shared memory)
    __shared__ uint4 *s_lv[kRedBlockLog + 1];
    if (tid <= kmax) s_lv[tid] = T.at(aa, l0 + tid, s0 >> tid);
    __syncthreads();
    int r = 0;                       // relative level of the current nodes
    uint32_t c = m;                  // their count
    while (r < kmax && (c > 32 || r == 0)) {
        const int d = kmax - r >= 2 ? 2 : 1;
        const uint32_t per = 1u << d;
        const uint32_t need = (c + per - 1) >> d;
        const uint4 *in = buf[(r >> 1) & 1];
        uint4 *out = buf[((r >> 1) + 1) & 1];
        if ((uint32_t)tid < need) {
            const uint32_t i0 = per * (uint32_t)tid;
            uint4 x[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                x[q] = make_uint4(0u, 0u, 0u, 0u);
                if (q < (int)per && i0 + q < c) x[q] = r == 0 ? __ldcg(s_lv[0] + i0 + q) : in[i0 + q];
            }
            const uint32_t c1 = (c + 1) >> 1;
            uint4 y0 = x[0], y1 = x[2];
            const uint4 h0 = hash_children32(x[0], x[1]);
            if (i0 + 1 < c) y0 = h0;
            uint4 *d1 = s_lv[r + 1];
            d1[i0 >> 1] = y0;
            if (d == 2) {
                const uint4 h1 = hash_children32(x[2], x[3]);
                if (i0 + 3 < c) y1 = h1;
                if ((i0 >> 1) + 1 < c1) d1[(i0 >> 1) + 1] = y1;
                uint4 z = y0;
                const uint4 hz = hash_children32(y0, y1);
                if ((i0 >> 1) + 1 < c1) z = hz;
                s_lv[r + 2][tid] = z;
                out[tid] = z;
            } else {
                out[tid] = y0;
            }
        }
        r += d;
        c = need;
        __syncthreads();
    }
    if (r < kmax && warp == 0) {
        // c <= 32 nodes of relative level r in buf: lane l holds node l
        uint4 z = (uint32_t)lane < c ? buf[(r >> 1) & 1][lane] : make_uint4(0u, 0u, 0u, 0u);
        for (int k = r + 1, step = 1; k <= kmax; ++k, step <<= 1) {
            const uint4 rr = shfl_down4(z, step);
            const uint32_t j = (uint32_t)lane >> (k - r);
            const uint32_t cp = (m + (1u << (k - 1)) - 1) >> (k - 1);     // nodes at level k-1
            if ((lane & (2 * step - 1)) == 0 && j < ((cp + 1) >> 1)) {
                if (2 * j + 1 < cp) z = hash_children32(z, rr);
                s_lv[k][j] = z;
            }
        }
    }
    __syncthreads();
}

// All levels of array aa above level l0 (its m nodes there, starting at node 0), block by block.
__device__ __noinline__ void reduce_up(const TreeRef &T, int aa, int l0, uint64_t m, uint4 *s_root) {
    const int top = T.levels(aa) - 1;
    while (l0 < top) {
        const int kmax = (top - l0) < kRedBlockLog ? (top - l0) : kRedBlockLog;
        for (uint64_t s0 = 0; s0 < m; s0 += (1u << kRedBlockLog)) {
            const uint64_t rest = m - s0;
            reduce_block(T, aa, l0, s0, (uint32_t)(rest < (1u << kRedBlockLog) ? rest : (1u << kRedBlockLog)),
                         kmax, s_root);
        }
        m = (m + (1ull << kmax) - 1) >> kmax;
        l0 += kmax;
    }
}

}  // namespace ckpt

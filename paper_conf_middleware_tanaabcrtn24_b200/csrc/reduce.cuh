// reduce.cuh -- latency-first interior levels for the finish kernel (finish.cuh).
//
// Alg. 1 lines 13-20, reading R13/R14: node j of level l+1 is
// Murmur3F(node 2j || node 2j+1, 32 B, seed 0), or node 2j promoted when it has no right
// sibling.  Any aligned block of 2^k nodes of a level is an exact subtree, so a CTA can reduce
// a block of up to 2048 nodes to its root on its own.  The levels kernel (levels.cuh) does it in
// passes of two levels through shared memory, which keeps lanes busy when there are many
// groups; here the goal is the shortest dependent chain, since the finish kernel's level work
// is small and sits at the end of the step:
//   * registers: each of the 512 threads takes 4 consecutive nodes and hashes them two levels up
//     (2 independent hashes, then 1);
//   * warp shuffles: the 32 results of a warp go 5 levels up (lane-halving);
//   * one barrier: the 16 warp results go the last 4 levels up in warp 0.
// 11 dependent hash latencies and one __syncthreads per 2048-node block; every node produced is
// stored at its place in the tree.
#pragma once
#include <cstdint>

#include "levels.cuh"
#include "mm32.cuh"

namespace ckpt {

constexpr int kRedBlockLog = 11;                 // nodes per block: 2^11 = 512 threads x 4
constexpr int kRedThreads = 512;

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

// Levels l0+1 .. l0+kmax (kmax <= 11) of the block of m <= 2048 level-l0 nodes of array aa
// starting at node s0 (s0 a multiple of 2^11); c_l = the block's node counts per level.
// Called by all 512 threads; s_root: 16 nodes of shared memory.
__device__ __noinline__ void reduce_block(const TreeRef &T, int aa, int l0, uint64_t s0, uint32_t m,
                                          int kmax, uint4 *s_root) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // the block's node count at relative level k
    auto cnt = [&](int k) -> uint32_t { return (m + (1u << k) - 1) >> k; };
    // ---- registers: levels 1 and 2 ----
    uint4 x[4];
    const uint32_t i0 = 4u * (uint32_t)tid;
    const uint4 *src = T.at(aa, l0, s0);
#pragma unroll
    for (int q = 0; q < 4; ++q) x[q] = i0 + q < m ? __ldcg(src + i0 + q) : make_uint4(0u, 0u, 0u, 0u);
    uint4 y0 = x[0], y1 = x[2];
    const uint4 h0 = hash_children32(x[0], x[1]), h1 = hash_children32(x[2], x[3]);
    if (i0 + 1 < m) y0 = h0;
    if (i0 + 3 < m) y1 = h1;
    uint4 z = y0;
    if (kmax >= 1) {
        uint4 *d = T.at(aa, l0 + 1, s0 >> 1);
        if (2 * tid < cnt(1)) d[2 * tid] = y0;
        if (2 * tid + 1 < cnt(1)) d[2 * tid + 1] = y1;
    }
    if (kmax >= 2) {
        const uint4 hz = hash_children32(y0, y1);
        if (2 * tid + 1 < cnt(1)) z = hz;
        if ((uint32_t)tid < cnt(2)) T.at(aa, l0 + 2, s0 >> 2)[tid] = z;
    }
    // ---- warp shuffles: levels 3..7 (lane l holds level-2 node 32*warp + l) ----
    for (int k = 3, step = 1; k <= 7 && k <= kmax; ++k, step <<= 1) {
        const uint4 r = shfl_down4(z, step);
        const uint32_t j = (32u * warp + lane) >> (k - 2);
        if ((lane & (2 * step - 1)) == 0 && j < cnt(k)) {
            if (2 * j + 1 < cnt(k - 1)) z = hash_children32(z, r);
            T.at(aa, l0 + k, s0 >> k)[j] = z;
        }
    }
    // ---- one barrier: levels 8..11 in warp 0 (lane w holds warp w's level-7 node) ----
    if (kmax >= 8) {
        if (lane == 0) s_root[warp] = z;
        __syncthreads();
        if (warp == 0) {
            uint4 w = lane < 16 ? s_root[lane] : make_uint4(0u, 0u, 0u, 0u);
            for (int k = 8, step = 1; k <= kmax; ++k, step <<= 1) {
                const uint4 r = shfl_down4(w, step);
                const uint32_t j = (uint32_t)lane >> (k - 7);
                if ((lane & (2 * step - 1)) == 0 && j < cnt(k)) {
                    if (2 * j + 1 < cnt(k - 1)) w = hash_children32(w, r);
                    T.at(aa, l0 + k, s0 >> k)[j] = w;
                }
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

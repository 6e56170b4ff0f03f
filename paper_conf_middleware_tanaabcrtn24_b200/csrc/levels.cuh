// levels.cuh -- K2: interior Merkle levels, several levels per launch.
//
// Paper: Alg. 1 lines 13-20 -- "for all node in level do in
// parallel: Tree(node) <- hash({left, right})", levels bottom-up; flattened
// array storage.  Reading R13: n_{l+1} = ceil(n_l/2), an odd last
// node is promoted unchanged, so any aligned group of 2^G nodes of level l is
// an exact subtree and a CTA can finish G levels of it in shared memory.
//
// One launch: CTA = one aligned group of kGroup nodes of level `ls` of one
// array -> levels ls+1 .. ls+kLog (written to global as they are formed).
// The last CTA to finish (atomic ticket) builds every remaining level of every
// array from L2 and then the top tree over the array roots (R15), so a whole
// tree takes one leaf launch + one level launch.
#pragma once
#include <cstdint>

#include "hash.cuh"

namespace ckpt {

constexpr int kLevelThreads = 512;
constexpr int kLog = 10;
constexpr int kGroup = 1 << kLog;       // nodes of level ls per CTA

struct LevelParams {
    uint4 *nodes;                 // whole tree storage
    const uint64_t *off;          // [level * n_arrays + a]: node index of array a's level
    const uint64_t *cnt;          // [level * n_arrays + a]: node count (0 above the array's root)
    const uint64_t *gbegin;       // [a]: first CTA of array a (prefix of ceil(cnt[ls][a]/kGroup))
    const uint64_t *level_base;   // [level]: node index of level (all arrays, concatenated)
    const uint64_t *level_total;  // [level]: nodes in level (all arrays)
    const uint32_t *height;       // [a]: number of levels of array a
    uint64_t top_off;             // node index of the top tree's level 0
    unsigned int *ticket;         // zero-initialised counter
    int n_arrays;
    int n_levels;                 // max height over arrays
    int ls;                       // start level of this launch
};

__device__ __forceinline__ int find_group_array(const uint64_t *gbegin, int n_arrays, uint64_t g) {
    int lo = 0, hi = n_arrays - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (gbegin[mid] <= g) lo = mid; else hi = mid - 1;
    }
    return lo;
}

__device__ __forceinline__ int find_level_array(const uint64_t *off_l, int n_arrays, uint64_t idx) {
    int lo = 0, hi = n_arrays - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (off_l[mid] <= idx) lo = mid; else hi = mid - 1;
    }
    return lo;
}

__global__ void __launch_bounds__(kLevelThreads) levels_kernel(LevelParams p) {
    __shared__ uint4 buf[kGroup];
    __shared__ unsigned int s_ticket;
    const int tid = threadIdx.x;
    const int na = p.n_arrays;
    {
        const int a = find_group_array(p.gbegin, na, blockIdx.x);
        const uint64_t g = blockIdx.x - p.gbegin[a];
        const uint64_t n0 = p.cnt[(uint64_t)p.ls * na + a];
        const uint64_t start = g * kGroup;
        int m = (int)((n0 - start) < (uint64_t)kGroup ? (n0 - start) : (uint64_t)kGroup);
        const uint4 *src = p.nodes + p.off[(uint64_t)p.ls * na + a] + start;
        for (int i = tid; i < m; i += kLevelThreads) buf[i] = src[i];
        const int h = (int)p.height[a];
        for (int k = 1; k <= kLog && p.ls + k < h; ++k) {
            const int mk = (m + 1) >> 1;
            __syncthreads();
            uint4 v[kGroup / 2 / kLevelThreads > 0 ? kGroup / 2 / kLevelThreads : 1];
#pragma unroll
            for (int r = 0; r < (kGroup / 2 + kLevelThreads - 1) / kLevelThreads; ++r) {
                const int j = tid + r * kLevelThreads;
                if (j < mk) v[r] = (2 * j + 1 < m) ? hash_children(buf[2 * j], buf[2 * j + 1]) : buf[2 * j];
            }
            __syncthreads();
            uint4 *dst = p.nodes + p.off[(uint64_t)(p.ls + k) * na + a] + (start >> k);
#pragma unroll
            for (int r = 0; r < (kGroup / 2 + kLevelThreads - 1) / kLevelThreads; ++r) {
                const int j = tid + r * kLevelThreads;
                if (j < mk) {
                    buf[j] = v[r];
                    dst[j] = v[r];
                }
            }
            m = mk;
        }
    }
    // ---- last CTA: remaining levels of every array, then the top tree ----
    __threadfence();
    __syncthreads();
    if (tid == 0) s_ticket = atomicAdd(p.ticket, 1u);
    __syncthreads();
    if (s_ticket != gridDim.x - 1) return;
    __threadfence();
    for (int l = p.ls + kLog + 1; l < p.n_levels; ++l) {
        const uint64_t total = p.level_total[l];
        const uint64_t base = p.level_base[l];
        const uint64_t *off_l = p.off + (uint64_t)l * na;
        const uint64_t *off_d = p.off + (uint64_t)(l - 1) * na;
        const uint64_t *cnt_d = p.cnt + (uint64_t)(l - 1) * na;
        for (uint64_t i = tid; i < total; i += kLevelThreads) {
            const int a = find_level_array(off_l, na, base + i);
            const uint64_t j = base + i - off_l[a];
            const uint64_t nd = cnt_d[a];
            const uint4 *c = p.nodes + off_d[a];
            uint4 v = __ldcg(c + 2 * j);
            if (2 * j + 1 < nd) v = hash_children(v, __ldcg(c + 2 * j + 1));
            p.nodes[base + i] = v;
        }
        __syncthreads();
    }
    // top tree: level 0 = array roots in array order
    for (int a = tid; a < na; a += kLevelThreads) {
        const int h = (int)p.height[a];
        p.nodes[p.top_off + a] = __ldcg(p.nodes + p.off[(uint64_t)(h - 1) * na + a]);
    }
    __syncthreads();
    uint64_t n = (uint64_t)na, cur = p.top_off;
    while (n > 1) {
        const uint64_t up = (n + 1) >> 1;
        for (uint64_t j = tid; j < up; j += kLevelThreads) {
            uint4 v = __ldcg(p.nodes + cur + 2 * j);
            if (2 * j + 1 < n) v = hash_children(v, __ldcg(p.nodes + cur + 2 * j + 1));
            p.nodes[cur + n + j] = v;
        }
        __syncthreads();
        cur += n;
        n = up;
    }
    if (tid == 0) *p.ticket = 0u;
}

}  // namespace ckpt

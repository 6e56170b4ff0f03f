// follow.cuh -- the follower of the fused pair launch: four warps per SM that run next to K1
// and do the post-leaf work of each tile as soon as K1 publishes the tile.
//
// K1 (leaf.cuh, leaf_pair_kernel) occupies every SM with three 8-warp CTAs of 72 registers,
// which leaves 2560 registers free in each of the SM's four sub-partitions: one 80-register warp
// each.  The follower grid (one 4-warp CTA per SM) is launched right after K1 with programmatic
// dependent launch, so its CTAs become resident while K1 runs and never take a slot from a K1
// warp (tools/probe_follow.py measures when they start).  K1's warps stay the only
// hashing warps; the follower spends the SM's spare issue slots and K1's spare HBM
// bandwidth (K1 is issue-bound at ~72 % of HBM peak).
//
// Work: K1 groups its pair-tasks in tiles of kTileTasks; the warp that completes a tile writes
// the tile's flagged chunk ids (tile_compact) and then releases tready[tile] = epoch.  The
// follower warps share a tile cursor: a warp waits for the cursor's tile (acquire) and takes
// jobs of kFollowJob flagged chunks from the tile's counter -- the element test of verify
// (reading R9: |(double)a_i - (double)b_i| > eps) into the hit count and hit mask
// of the chunk's tile slot (mark.cuh) -- and moves the cursor on once the tile is handed out.
// After K1 the ordered chunk list, the scan and the emit read the tile slots (compare.cuh,
// premarked mode).  DESIGN.md section 7 has the measurements.
#pragma once
#include <cstdint>

#include "leaf.cuh"
#include "mark.cuh"

namespace ckpt {

constexpr int kFollowWarps = 4;               // one warp per SM sub-partition
constexpr uint32_t kFollowMaxChunk = 32768;   // K1 runs at 72 registers below this chunk size
constexpr int kFollowJob = 4;                 // flagged chunks per job
constexpr int kFollowMarkBatch = 4;           // mark_chunk loads in flight per lane (4 x 16 B x 2)

struct FollowParams {
    const LeafArray *arrays;      // K1's table: A's m arrays, then B's m arrays (device), or
    LeafArray inl[kLeafInline];   // inline when 2m <= kLeafInline
    int n_arrays;                 // 2m
    int m;
    uint32_t chunk;               // C bytes
    uint32_t per;                 // elements per chunk
    uint32_t groups;              // mask groups (32 words of 32 bits) per chunk
    double eps;
    const uint32_t *tagg;         // K1: flagged chunks per tile
    const uint64_t *tids;         // K1: the tile's flagged chunk ids, ascending
    const uint32_t *tready;       // K1: epoch once tile t is published
    uint32_t epoch;
    uint32_t n_tiles;
    uint64_t n_pair;              // pair-tasks (A's tasks)
    unsigned int *tsub;           // [n_tiles + 2] job counters, finished warps, tile cursor
                                  // (0 at launch, reset by the last warp)
    uint32_t *scnt;               // [tile slot] hits of the slot's chunk
    uint32_t *smask;              // [tile slot][groups * 32] hit bits (element-contiguous words)
};

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint64_t global_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// Mark the flagged chunk in tile slot `slot` (global chunk id g of tree A).
template <int DT>
__device__ __forceinline__ void follow_mark(const FollowParams &p, const LeafArray *arrays,
                                            uint64_t slot, int lane) {
    constexpr int ESZ = DT == 0 ? 4 : 8;
    const uint64_t g = __ldcg(reinterpret_cast<const unsigned long long *>(p.tids) + slot);
    int lo = 0, hi = p.m - 1;                 // A's array holding chunk g
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (arrays[mid].chunk_base <= g) lo = mid; else hi = mid - 1;
    }
    const LeafArray &A = arrays[lo];
    const uint64_t e0 = (g - A.chunk_base) * p.per;
    const uint64_t n = A.nbytes / ESZ;
    const uint64_t len = (n - e0) < p.per ? n - e0 : p.per;
    const uint8_t *pa = A.data + e0 * ESZ;
    const uint8_t *pb = arrays[lo + p.m].data + e0 * ESZ;
    const uint32_t c = mark_chunk<DT, kFollowMarkBatch>(pa, pb, len, p.eps,
                                                        p.smask + slot * p.groups * 32, lane);
    if (lane == 0) p.scnt[slot] = c;
}

template <int DT>
__global__ void __launch_bounds__(kFollowWarps * 32, 6) follow_kernel(const __grid_constant__ FollowParams p) {
    // no griddepcontrol.wait here: the follower runs concurrently with K1 (its programmatic
    // primary) and synchronises with it through the tile flags only.  Every warp works alone.
    const int lane = threadIdx.x & 31;
    const LeafArray *arrays = p.n_arrays <= kLeafInline ? p.inl : p.arrays;
    unsigned int *tcur = p.tsub + p.n_tiles + 1;    // first tile that may still hold jobs
    constexpr uint64_t kTimeoutNs = 60ull * 1000000000ull;
    uint32_t t = 0;
    for (;;) {
        if (lane == 0) {
            const uint32_t c = *reinterpret_cast<volatile unsigned int *>(tcur);
            t = c > t ? c : t;
        }
        t = __shfl_sync(0xffffffffu, t, 0);
        if (t >= p.n_tiles) break;
        if (lane == 0 && ld_acquire_u32(p.tready + t) != p.epoch) {
            const uint64_t t0 = global_ns();
            unsigned int nap = 256;
            do {
                __nanosleep(nap);
                nap = nap < 4096 ? 2 * nap : nap;
                if (global_ns() - t0 > kTimeoutNs) __trap();   // K1 never published the tile
            } while (ld_acquire_u32(p.tready + t) != p.epoch);
        }
        __syncwarp();   // lane 0's acquire, then every lane's loads
        const uint32_t n_flag = __ldcg(p.tagg + t);
        const uint32_t n_jobs = (n_flag + kFollowJob - 1) / kFollowJob;
        unsigned int j = n_jobs;
        if (n_jobs && lane == 0) j = atomicAdd(p.tsub + t, 1u);
        j = __shfl_sync(0xffffffffu, j, 0);
        if (j < n_jobs) {
            const uint32_t k0 = j * kFollowJob;
            const uint32_t k1 = (k0 + kFollowJob) < n_flag ? k0 + kFollowJob : n_flag;
            for (uint32_t k = k0; k < k1; ++k)
                follow_mark<DT>(p, arrays, (uint64_t)t * kTileTasks * 32 + k, lane);
            continue;
        }
        if (lane == 0) atomicMax(tcur, t + 1);       // tile t is handed out: move every warp on
        ++t;
    }
    // K1 complete (and its memory visible) before this grid completes, so the next kernel on the
    // stream sees both; then the last warp resets the counters for the next launch
    asm volatile("griddepcontrol.wait;" ::: "memory");
    unsigned int d = 0;
    if (lane == 0) d = atomicAdd(p.tsub + p.n_tiles, 1u);
    d = __shfl_sync(0xffffffffu, d, 0);
    if (d == gridDim.x * kFollowWarps - 1) {
        for (uint32_t k = lane; k <= p.n_tiles + 1; k += 32) p.tsub[k] = 0u;
    }
}

}  // namespace ckpt

// finish.cuh -- K5: everything the fused pair path does after the leaf kernel, ONE launch.
//
// K1 (leaf.cuh, PAIR mode) leaves the leaves of both trees and, per tile of 4096 chunks,
// the ascending ids of the chunks whose digests differ (the BFS of P:555-566 at start level
// 0).  What remains is latency-bound: the interior levels of both trees (Alg. 1)
// and the element test of the flagged chunks with the ordered output.  Doing it
// inside K1 was measured 2-4x costlier than its instruction count (profiles/r2/inK1_finish_ab.md:
// K1 is issue-bound at its register-limited 24 warps per SM, and latency-bound side work there
// idles warp slots nothing else can fill), so it runs here, at full occupancy, with both
// parts in one grid instead of a levels kernel on a side stream plus three verify kernels:
//
//  * tickets [0, n_level_ctas): level groups of both trees (levels.cuh, levels_cta: 2048-node
//    groups in shared memory, the last CTA of a tree builds the rest and the top tree);
//  * the following tickets: verify tiles of kFinTile consecutive positions of the flagged
//    chunk list, in list order.  A tile marks its chunks (one warp per chunk: binary64
//    |a-b| > eps, R11, hit bits to the work buffer), scans their hit counts, finds its output
//    offset by a decoupled look-back over the preceding tiles, and writes the element ids --
//    a single pass, no grid-wide step between marking and emitting.
//
// Tickets are drawn in order by co-resident CTAs, so a look-back only waits on tiles that
// running CTAs already hold.
#pragma once
#include <cstdint>

#include "compare.cuh"
#include "hash.cuh"
#include "levels.cuh"
#include "mark.cuh"

namespace ckpt {

constexpr int kFinThreads = kLevelThreads;         // 512 (the level groups' CTA shape)
constexpr int kFinWarps = kFinThreads / 32;
constexpr int kFinPerWarp = 2;                     // list positions per warp and tile
constexpr int kFinTile = kFinWarps * kFinPerWarp;  // 32 flagged chunks per verify tile

struct FinishParams {
    LevelBatch lv;                // both trees' level groups (lv.cta_begin[lv.n] CTAs)
    VerifyParams v;               // tile mode (v.tagg != null): the list comes from K1's tiles
    unsigned long long *ticket;   // 0 on entry; the last draw resets it
    unsigned int n_level;         // level tickets
};

__device__ __forceinline__ uint64_t fin_draw(unsigned long long *ticket, uint64_t n_total,
                                             uint64_t *s_t) {
    __syncthreads();                                   // the previous item is done with smem
    if (threadIdx.x == 0) {
        const uint64_t t = atomicAdd(ticket, 1ull);
        if (t == n_total + gridDim.x - 1) *ticket = 0ull;   // the last draw of the launch
        *s_t = t;
    }
    __syncthreads();
    return *s_t;
}

constexpr size_t kFinSmem = (size_t)kFinWarps * 1024 * 2 > (size_t)kLevelSmem
                               ? (size_t)kFinWarps * 1024 * 2 : (size_t)kLevelSmem;

template <int DT>
__global__ void __launch_bounds__(kFinThreads, 2) finish_kernel(const __grid_constant__ FinishParams P) {
    pdl_enter();
    constexpr int ESZ = DT == 0 ? 4 : 8;
    extern __shared__ __align__(16) uint4 fin_sm[];              // kFinSmem: level groups / emit scratch
    __shared__ uint32_t s_tpre[kVerifyMaxTiles + 1];             // K1 tile prefix (list positions)
    __shared__ uint32_t s_cnt[kFinTile], s_ex[kFinTile], s_len[kFinTile];
    __shared__ uint64_t s_gb[kFinTile];
    __shared__ const uint8_t *s_pa[kFinTile], *s_pb[kFinTile];
    __shared__ uint32_t s_sum;
    __shared__ uint64_t s_t;
    __shared__ unsigned int s_ticket;
    const VerifyParams &p = P.v;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // the flagged-chunk list: K1's per-tile compaction, prefixed once per CTA
    tile_prefix<kFinThreads>(p, s_tpre);
    const uint64_t total = s_tpre[p.n_tiles];
    const uint64_t n_list = total < p.chunks_cap ? total : p.chunks_cap;
    const uint64_t n_vt = (n_list + kFinTile - 1) / kFinTile;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *p.n_chunks_out = total;
        if (n_vt == 0) *p.count = 0;
    }
    const uint64_t n_total = P.n_level + n_vt;
    for (uint64_t t = fin_draw(P.ticket, n_total, &s_t); t < n_total; t = fin_draw(P.ticket, n_total, &s_t)) {
        if (t < P.n_level) {
            levels_cta(P.lv, (unsigned int)t, fin_sm, s_ticket);
            continue;
        }
        // ---------------- verify tile vt: list positions [q0, q0 + kFinTile) ----------------
        const uint64_t vt = t - P.n_level;
        const uint64_t q0 = vt * kFinTile;
        const uint32_t nq = (uint32_t)((n_list - q0) < (uint64_t)kFinTile ? (n_list - q0) : kFinTile);
        if (threadIdx.x < kFinTile) {                  // locate the tile's chunks, one thread each
            const uint32_t j = threadIdx.x;
            const uint8_t *pa = nullptr, *pb = nullptr;
            uint64_t len = 0, gb = 0;
            if (j < nq) {
                const uint64_t g = tile_chunk(p, s_tpre, q0 + j);
                p.list_out[q0 + j] = g;
                verify_locate_g(p, g, ESZ, pa, pb, len, gb);
            }
            s_pa[j] = pa;
            s_pb[j] = pb;
            s_len[j] = (uint32_t)len;
            s_gb[j] = gb;
        }
        __syncthreads();
        for (int k = 0; k < kFinPerWarp; ++k) {        // mark: one warp per chunk
            const uint32_t j = warp * kFinPerWarp + k;
            uint32_t c = 0;
            if (j < nq)
                c = mark_chunk<DT>(s_pa[j], s_pb[j], s_len[j], p.eps, p.mask + (q0 + j) * p.groups * 32, lane);
            if (lane == 0) s_cnt[j] = c;
        }
        __syncthreads();
        if (warp == 0) {                               // the tile's exclusive prefix of hit counts
            uint32_t tot;
            const uint32_t ex = warp_excl_scan_u32(lane < kFinTile ? s_cnt[lane] : 0u, lane, tot);
            if (lane < kFinTile) s_ex[lane] = ex;
            if (lane == 0) s_sum = tot;
        }
        __syncthreads();
        const uint64_t excl = cta_lookback<kFinThreads>(p.states, vt, s_sum, p.epoch);
        if (threadIdx.x == 0 && vt == n_vt - 1) *p.count = excl + s_sum;
        // ids: each warp writes its own chunks' (ascending, coalesced)
        uint16_t *s_off = reinterpret_cast<uint16_t *>(fin_sm) + warp * 1024;
        for (int k = 0; k < kFinPerWarp; ++k) {
            const uint32_t j = warp * kFinPerWarp + k;
            if (j >= nq || s_cnt[j] == 0) continue;    // warp-uniform
            uint64_t pos = excl + s_ex[j];
            const uint32_t groups = (s_len[j] + 1023) / 1024;
            const uint32_t *mq = p.mask + (q0 + j) * p.groups * 32 + lane;
            for (uint32_t g = 0; g < groups; ++g)
                pos += emit_words(__ldcs(mq + g * 32), s_gb[j] + (uint64_t)g * 1024, pos, p.out, p.cap, lane,
                                  s_off);
        }
    }
}

}  // namespace ckpt

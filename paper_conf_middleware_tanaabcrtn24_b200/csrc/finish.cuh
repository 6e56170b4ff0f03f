// finish.cuh -- K5: everything the fused pair path does after the leaves, ONE launch that
// runs alongside the leaf kernel's tail.
//
// K1 (leaf.cuh, PAIR mode) leaves the leaves of both trees and, per tile of 128 pair-tasks
// (4096 chunks), the ascending ids of the chunks whose digests differ (the BFS of P:555-566
// at start level 0), publishing each finished tile with a release flag (tdone[tile] = the
// launch's epoch).  What remains is latency-bound: the interior levels of both trees
// (Alg. 1) and the element test of the flagged chunks with the ordered output
// (P:568-578).  Doing it inside K1 was measured 2-4x costlier than its instruction count
// (profiles/r2/inK1_finish_ab.md: K1 is issue-bound at its register-limited 24 warps per SM,
// and latency-bound side work there idles warp slots nothing else can fill).  Here it runs in
// its own grid, launched with programmatic dependent launch and WITHOUT waiting for K1 to
// complete: its CTAs take the SM slots K1's CTAs free during K1's tail (the last ~10% of K1,
// where warps run out of tasks) and consume K1's tiles as they are published.
//
//  * tickets [0, n_tiles): verify item k = K1 tile k.  Wait for tdone[k]; mark the tile's
//    flagged chunks (one warp per chunk: binary64 |a-b| > eps, R11; hit bits to the work
//    buffer), scan their hit counts in the CTA, then a decoupled look-back over the preceding
//    items gives both the tile's first chunk-list position and its first element-id position;
//    write the chunk ids and the element ids (ascending, coalesced).
//  * tickets [n_tiles, n_tiles + n_level): level groups of both trees, each after the K1
//    tiles holding its leaves are published: 2048 leaves of one array per CTA reduced 11
//    levels up (reduce.cuh: registers, shuffles, one barrier); the last group of an array
//    builds the array's remaining levels, the last array of a tree the top tree (R15).
//
// Tickets are drawn in order by running CTAs and every wait is on work that K1 (resident from
// its start) or an earlier ticket's CTA completes, so nothing waits on a CTA that cannot run.
#pragma once
#include <cstdint>

#include "compare.cuh"
#include "hash.cuh"
#include "levels.cuh"
#include "mark.cuh"
#include "reduce.cuh"

namespace ckpt {

constexpr int kFinThreads = kLevelThreads;         // 512 (the level groups' CTA shape)
constexpr int kFinWarps = kFinThreads / 32;
constexpr int kTileIdsFin = 4096;                  // chunk slots per K1 tile (kTileTasks * 32)
// dynamic shared memory: per-chunk hit counts of a tile (16 KB) + per-warp emit scratch
// (2 KB each), or the level groups' kLevelSmem
constexpr size_t kFinSmemVerify = (size_t)kTileIdsFin * 4 + (size_t)kFinWarps * 2048;
constexpr size_t kFinSmem = kFinSmemVerify > (size_t)kLevelSmem ? kFinSmemVerify : (size_t)kLevelSmem;

struct FinishParams {
    LevelBatch lv;                // both trees' level groups (lv.cta_begin[lv.n] CTAs)
    VerifyParams v;               // tagg / tids / n_tiles: K1's tiles; mask: per tile slot
    unsigned long long *ticket;   // 0 on entry; the last draw resets it
    unsigned int n_level;         // level tickets
    const uint32_t *tdone;        // [n_tiles] K1's tile flags
    uint32_t tepoch;              // this pair compare's tag in tdone
    uint64_t *states_c;           // look-back states of the chunk-list positions (p.states: element ids)
    unsigned int *lctr;           // [2 * na + 2] level arrivals per (tree, array), per tree; 0 between launches
};

__device__ __forceinline__ unsigned int atom_add_acq_rel_u32(unsigned int *p, unsigned int v) {
    unsigned int old;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}

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

// Thread 0 waits (acquire, growing sleep) until K1 published tiles [lo, hi]; then a barrier.
__device__ __forceinline__ void fin_wait_tiles(const FinishParams &P, uint64_t lo, uint64_t hi) {
    if (threadIdx.x == 0) {
        unsigned int nap = 64;
        for (uint64_t k = lo; k <= hi; ++k) {
            for (;;) {
                uint32_t v;
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(P.tdone + k) : "memory");
                if (v == P.tepoch) break;
                __nanosleep(nap);
                nap = nap < 2048u ? 2u * nap : 2048u;
            }
        }
    }
    __syncthreads();
}

template <int DT>
__global__ void __launch_bounds__(kFinThreads, 2) finish_kernel(const __grid_constant__ FinishParams P) {
    // no griddepcontrol.wait: this grid runs while K1 still does (see above); its successor
    // waits for it as usual
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    constexpr int ESZ = DT == 0 ? 4 : 8;
    extern __shared__ __align__(16) uint4 fin_sm[];
    __shared__ uint32_t s_w[kFinWarps];
    __shared__ uint64_t s_t;
    __shared__ unsigned int s_ticket;
    const VerifyParams &p = P.v;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t n_tiles = p.n_tiles;
    const uint64_t n_total = n_tiles + P.n_level;
    for (uint64_t t = fin_draw(P.ticket, n_total, &s_t); t < n_total; t = fin_draw(P.ticket, n_total, &s_t)) {
        if (t >= n_tiles) {
            // ------------------------------ a level group ------------------------------
            const unsigned int cta = (unsigned int)(t - n_tiles);
            int ti = 0;
            while (ti + 1 < P.lv.n && cta >= P.lv.cta_begin[ti + 1]) ++ti;
            const LevelParams &lp = P.lv.t[ti];
            const uint8_t *mb = lp.inl >= 0 ? reinterpret_cast<const uint8_t *>(P.lv.blob + lp.inl) : lp.meta;
            const uint64_t *gbegin = reinterpret_cast<const uint64_t *>(mb + lp.o_g);
            const uint64_t *cnt0 = reinterpret_cast<const uint64_t *>(mb + lp.o_cnt);   // level 0
            const int na = lp.n_arrays;
            const uint64_t gid = cta - P.lv.cta_begin[ti];
            const int a = find_le(gbegin, na, gid);
            // pair-tasks (32 chunks of one array each, array-major) holding the group's leaves
            uint64_t tb = 0;
            for (int k = 0; k < a; ++k) tb += (cnt0[k] + 31) / 32;
            const uint64_t g = gid - gbegin[a];
            const uint64_t c_lo = g * kGroup;
            const uint64_t c_hi = (c_lo + kGroup < cnt0[a] ? c_lo + kGroup : cnt0[a]) - 1;
            fin_wait_tiles(P, (tb + c_lo / 32) / kTileTasks, (tb + c_hi / 32) / kTileTasks);
            if (lp.inl >= 0 && gid == 0) {
                // publish the inline tables to device memory for later BFS launches
                uint64_t *dst = reinterpret_cast<uint64_t *>(lp.meta);
                for (uint32_t w = threadIdx.x; w < lp.meta_words; w += kFinThreads) dst[w] = P.lv.blob[lp.inl + w];
            }
            TreeRef T;
            T.nodes = lp.nodes;
            T.off = reinterpret_cast<const uint64_t *>(mb + lp.o_off);
            T.cnt = cnt0;
            T.height = reinterpret_cast<const uint32_t *>(mb + lp.o_h);
            T.top_off = lp.top_off;
            T.na = na;
            uint4 *s_root = fin_sm;
            const int H = (int)T.height[a];
            if (H > 1)
                reduce_block(T, a, 0, c_lo, (uint32_t)(c_hi + 1 - c_lo), H - 1 < kRedBlockLog ? H - 1 : kRedBlockLog, s_root);
            if (H - 1 > kRedBlockLog) {
                // the last group of the array builds the array's remaining levels
                const uint32_t n_g = (uint32_t)((cnt0[a] + kGroup - 1) / kGroup);     // the array's groups
                if (threadIdx.x == 0) {
                    unsigned int *c = P.lctr + (uint32_t)ti * (uint32_t)na + (uint32_t)a;
                    const unsigned int old = atom_add_acq_rel_u32(c, 1u);
                    s_ticket = old;
                    if (old == n_g - 1) *c = 0u;
                }
                __syncthreads();
                if (s_ticket != n_g - 1) continue;
                reduce_up(T, a, kRedBlockLog, T.count(a, kRedBlockLog), s_root);
            }
            // the array root is final: it is level-0 node a of the top tree; the last array
            // of the tree builds the top
            if (threadIdx.x == 0) {
                *T.at(na, 0, (uint64_t)a) = __ldcg(T.at(a, H - 1, 0));
                unsigned int *c = P.lctr + 2 * (uint32_t)na + (uint32_t)ti;
                const unsigned int old = atom_add_acq_rel_u32(c, 1u);
                s_ticket = old;
                if (old == (unsigned int)na - 1) *c = 0u;
            }
            __syncthreads();
            if (s_ticket != (unsigned int)na - 1) continue;
            reduce_up(T, na, 0, (uint64_t)na, s_root);
            continue;
        }
        // ------------------------------ verify item k ------------------------------
        const uint64_t k = t;
        fin_wait_tiles(P, k, k);
        const uint32_t n = __ldcg(p.tagg + k);
        uint32_t *s_cnt = reinterpret_cast<uint32_t *>(fin_sm);           // [kTileIdsFin]
        const uint64_t *ids = p.tids + k * kTileIdsFin;
        for (uint32_t j = warp; j < n; j += kFinWarps) {                  // mark: a warp per chunk
            const uint64_t g = __ldcg(reinterpret_cast<const unsigned long long *>(ids) + j);
            const uint8_t *pa, *pb;
            uint64_t len, gb;
            verify_locate_g(p, g, ESZ, pa, pb, len, gb);
            const uint32_t c = mark_chunk<DT>(pa, pb, len, p.eps, p.mask + (k * kTileIdsFin + j) * p.groups * 32, lane);
            if (lane == 0) s_cnt[j] = c;
        }
        __syncthreads();
        // exclusive prefix of the hit counts over the tile's chunks (8 per thread)
        constexpr int kPer = kTileIdsFin / kFinThreads;
        uint32_t v[kPer], sum = 0;
        const uint32_t j0 = threadIdx.x * kPer;
#pragma unroll
        for (int i = 0; i < kPer; ++i) {
            v[i] = j0 + i < n ? s_cnt[j0 + i] : 0u;
            sum += v[i];
        }
        uint32_t wtot;
        uint32_t ex = warp_excl_scan_u32(sum, lane, wtot);
        if (lane == 0) s_w[warp] = wtot;
        __syncthreads();
        uint32_t hits = 0;
#pragma unroll
        for (int w = 0; w < kFinWarps; ++w) {
            const uint32_t x = s_w[w];
            if (w < warp) ex += x;
            hits += x;
        }
#pragma unroll
        for (int i = 0; i < kPer; ++i) {
            if (j0 + i < n) s_cnt[j0 + i] = ex;                // now: first hit of chunk j inside the tile
            ex += v[i];
        }
        __syncthreads();
        // the tile's place: chunk-list positions and element-id positions of all earlier tiles
        const uint64_t excl_c = cta_lookback<kFinThreads>(P.states_c, k, n, p.epoch);
        const uint64_t excl_h = cta_lookback<kFinThreads>(p.states, k, hits, p.epoch);
        const uint64_t cap_c = p.chunks_cap;
        if (threadIdx.x == 0) {
            if (k == n_tiles - 1) {
                *p.n_chunks_out = excl_c + n;
                if (excl_c + n <= cap_c) *p.count = excl_h + hits;
            }
            // the chunk-list capacity cuts this tile: the element ids are those of listed chunks
            if (excl_c < cap_c && cap_c < excl_c + n) *p.count = excl_h + s_cnt[cap_c - excl_c];
        }
        const uint32_t n_listed = excl_c >= cap_c ? 0u : (uint32_t)((cap_c - excl_c) < n ? (cap_c - excl_c) : n);
        for (uint32_t j = threadIdx.x; j < n_listed; j += kFinThreads)
            p.list_out[excl_c + j] = __ldcg(reinterpret_cast<const unsigned long long *>(ids) + j);
        uint16_t *s_off = reinterpret_cast<uint16_t *>(reinterpret_cast<uint8_t *>(fin_sm) + kTileIdsFin * 4) + warp * 1024;
        for (uint32_t j = warp; j < n_listed; j += kFinWarps) {           // ids: a warp per chunk
            const uint32_t c0 = s_cnt[j];
            const uint32_t c1 = j + 1 < n ? s_cnt[j + 1] : hits;
            if (c1 == c0) continue;                                       // warp-uniform
            const uint64_t g = __ldcg(reinterpret_cast<const unsigned long long *>(ids) + j);
            const uint8_t *pa, *pb;
            uint64_t len, gb;
            verify_locate_g(p, g, ESZ, pa, pb, len, gb);
            uint64_t pos = excl_h + c0;
            const uint32_t groups = (uint32_t)((len + 1023) / 1024);
            const uint32_t *mq = p.mask + (k * kTileIdsFin + j) * p.groups * 32 + lane;
            for (uint32_t gr = 0; gr < groups; ++gr)
                pos += emit_words(__ldcs(mq + gr * 32), gb + (uint64_t)gr * 1024, pos, p.out, p.cap, lane, s_off);
        }
    }
}

}  // namespace ckpt

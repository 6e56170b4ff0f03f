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
//  * tickets [0, n_level): level groups of both trees, each after the K1 tiles holding its
//    leaves are published: 2048 leaves of one array per CTA reduced 11 levels up (reduce.cuh);
//    the last group of an array builds the array's remaining levels, the last array of a tree
//    the top tree (R15).  These overlap K1's tail.
//  * the following tickets: verify blocks of kFinBlock consecutive positions of the flagged
//    chunk list, once every K1 tile is published (the list is K1's per-tile compaction,
//    prefixed in shared memory).  A block marks its chunks (one warp per chunk: binary64
//    |a-b| > eps, R11; hit bits to the work buffer), scans their hit counts, finds its output
//    offset by a decoupled look-back over the preceding blocks and writes the element ids
//    (ascending, coalesced) -- a single pass.
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

constexpr int kFinThreads = kRedThreads;           // 128: fits beside K1's CTAs as they retire
constexpr int kFinWarps = kFinThreads / 32;
constexpr uint64_t kFinGroup = 1u << kRedBlockLog;  // leaves per level item
constexpr int kFinPerWarp = 4;                     // flagged chunks per warp and verify block
constexpr int kFinBlock = kFinWarps * kFinPerWarp; // 16
// dynamic shared memory: 2 x 512 nodes for the level blocks, or 2 KB of emit scratch per warp
constexpr size_t kFinSmem = (size_t)kFinWarps * 2048 > (size_t)2 * kRedThreads * 16
                                ? (size_t)kFinWarps * 2048 : (size_t)2 * kRedThreads * 16;

struct FinishParams {
    LevelBatch lv;                // both trees' level groups (lv.cta_begin[lv.n] CTAs)
    VerifyParams v;               // tagg / tids / n_tiles: K1's tiles; mask: per list position
    unsigned long long *ticket;   // 0 on entry; the last draw resets it
    unsigned int n_level;         // level tickets
    const uint32_t *tdone;        // [n_tiles] K1's tile flags
    uint32_t tepoch;              // this pair compare's tag in tdone
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

// Wait until K1 published tiles [lo, hi]: the CTA's threads poll the flags in parallel with
// relaxed loads (a sequential acquire per tile would cost one L2 round trip each), then one
// acquire fence orders everything the flags published before this CTA's reads.
__device__ __forceinline__ void fin_wait_tiles(const FinishParams &P, uint64_t lo, uint64_t hi) {
    __shared__ int s_pending;
    unsigned int nap = 64;
    for (;;) {
        int mine = 0;
        for (uint64_t k = lo + threadIdx.x; k <= hi; k += blockDim.x) {
            uint32_t v;
            asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(P.tdone + k) : "memory");
            mine |= v != P.tepoch;
        }
        if (threadIdx.x == 0) s_pending = 0;
        __syncthreads();
        if (mine) s_pending = 1;
        __syncthreads();
        if (!s_pending) break;
        __nanosleep(nap);
        nap = nap < 2048u ? 2u * nap : 2048u;
    }
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    __syncthreads();
}

template <int DT>
__global__ void __launch_bounds__(kFinThreads, 8) finish_kernel(const __grid_constant__ FinishParams P) {
    // no griddepcontrol.wait: this grid runs while K1 still does (see above); its successor
    // waits for it as usual
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    constexpr int ESZ = DT == 0 ? 4 : 8;
    extern __shared__ __align__(16) uint4 fin_sm[];
    __shared__ uint32_t s_tpre[kVerifyMaxTiles + 1];             // K1 tile prefix (list positions)
    __shared__ uint32_t s_cnt[kFinBlock], s_len[kFinBlock];
    __shared__ uint64_t s_gb[kFinBlock];
    __shared__ const uint8_t *s_pa[kFinBlock], *s_pb[kFinBlock];
    __shared__ uint32_t s_ex[kFinBlock], s_sum;
    __shared__ uint64_t s_t;
    __shared__ unsigned int s_ticket;
    const VerifyParams &p = P.v;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    bool listed = false;                      // s_tpre holds the tile prefix
    uint64_t n_list = 0, n_vb = 0;
    for (;;) {
        __syncthreads();                      // the previous item is done with shared memory
        if (threadIdx.x == 0) s_t = atomicAdd(P.ticket, 1ull);
        __syncthreads();
        const uint64_t t = s_t;
        if (t < P.n_level) {
            // ------------------------------ a level group ------------------------------
            // both trees have the same shape: the first half of the level tickets is run A's
            const unsigned int half = P.n_level / 2;
            const int ti = t >= half ? 1 : 0;
            uint64_t gid = ti ? t - half : t;
            const LevelParams &lp = P.lv.t[ti];
            const uint8_t *mb = lp.inl >= 0 ? reinterpret_cast<const uint8_t *>(P.lv.blob + lp.inl) : lp.meta;
            const uint64_t *cnt0 = reinterpret_cast<const uint64_t *>(mb + lp.o_cnt);   // level 0
            const int na = lp.n_arrays;
            // the array of group gid (blocks of kFinGroup leaves, arrays in order), and the
            // pair-tasks (32 chunks of one array each, array-major) before it
            int a = 0;
            uint64_t tb = 0;
            for (;; ++a) {
                const uint64_t ng = (cnt0[a] + kFinGroup - 1) / kFinGroup;
                if (gid < ng || a == na - 1) break;
                gid -= ng;
                tb += (cnt0[a] + 31) / 32;
            }
            const uint64_t c_lo = gid * kFinGroup;
            const uint64_t c_hi = (c_lo + kFinGroup < cnt0[a] ? c_lo + kFinGroup : cnt0[a]) - 1;
            fin_wait_tiles(P, (tb + c_lo / 32) / kTileTasks, (tb + c_hi / 32) / kTileTasks);
            if (lp.inl >= 0 && a == 0 && gid == 0) {
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
            const int H = (int)T.height[a];
            if (H > 1)
                reduce_block(T, a, 0, c_lo, (uint32_t)(c_hi + 1 - c_lo), H - 1 < kRedBlockLog ? H - 1 : kRedBlockLog, fin_sm);
            if (H - 1 > kRedBlockLog) {
                // the last group of the array builds the array's remaining levels
                const uint32_t n_g = (uint32_t)((cnt0[a] + kFinGroup - 1) / kFinGroup);
                if (threadIdx.x == 0) {
                    unsigned int *c = P.lctr + (uint32_t)ti * (uint32_t)na + (uint32_t)a;
                    const unsigned int old = atom_add_acq_rel_u32(c, 1u);
                    s_ticket = old;
                    if (old == n_g - 1) *c = 0u;
                }
                __syncthreads();
                if (s_ticket != n_g - 1) continue;
                reduce_up(T, a, kRedBlockLog, T.count(a, kRedBlockLog), fin_sm);
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
            reduce_up(T, na, 0, (uint64_t)na, fin_sm);
            continue;
        }
        // -------- verify: blocks of kFinBlock consecutive positions of the flagged list --------
        if (!listed) {
            // every tile published: the list is K1's per-tile compaction, prefixed here
            fin_wait_tiles(P, 0, p.n_tiles - 1);
            tile_prefix<kFinThreads>(p, s_tpre);
            const uint64_t total = s_tpre[p.n_tiles];
            n_list = total < p.chunks_cap ? total : p.chunks_cap;
            n_vb = (n_list + kFinBlock - 1) / kFinBlock;
            listed = true;
            if (threadIdx.x == 0 && t == P.n_level) {
                *p.n_chunks_out = total;
                if (n_vb == 0) *p.count = 0;
            }
        }
        if (t >= P.n_level + n_vb) {
            // the last of the launch's final draws resets the ticket
            if (threadIdx.x == 0 && t == P.n_level + n_vb + gridDim.x - 1) *P.ticket = 0ull;
            break;
        }
        const uint64_t vb = t - P.n_level;
        const uint64_t q0 = vb * kFinBlock;
        const uint32_t nq = (uint32_t)((n_list - q0) < (uint64_t)kFinBlock ? (n_list - q0) : kFinBlock);
        if (threadIdx.x < kFinBlock) {               // locate the block's chunks, one thread each
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
        for (int k = 0; k < kFinPerWarp; ++k) {      // mark: warp w takes positions w, w+4, ...
            const uint32_t j = (uint32_t)(warp + kFinWarps * k);
            uint32_t c = 0;
            if (j < nq)
                c = mark_chunk<DT>(s_pa[j], s_pb[j], s_len[j], p.eps, p.mask + (q0 + j) * p.groups * 32, lane);
            if (lane == 0) s_cnt[j] = c;
        }
        __syncthreads();
        if (warp == 0) {                              // the block's exclusive prefix of hit counts
            uint32_t tot;
            const uint32_t ex = warp_excl_scan_u32(lane < kFinBlock ? s_cnt[lane] : 0u, lane, tot);
            if (lane < kFinBlock) s_ex[lane] = ex;
            if (lane == 0) s_sum = tot;
        }
        __syncthreads();
        const uint64_t excl = cta_lookback<kFinThreads>(p.states, vb, s_sum, p.epoch);
        if (threadIdx.x == 0 && vb == n_vb - 1) *p.count = excl + s_sum;
        for (int k = 0; k < kFinPerWarp; ++k) {      // ids: warp w writes its chunks'
            const uint32_t j = (uint32_t)(warp + kFinWarps * k);
            if (j >= nq || s_cnt[j] == 0) continue;   // warp-uniform
            uint16_t *s_off = reinterpret_cast<uint16_t *>(fin_sm) + warp * 1024;
            uint64_t pos = excl + s_ex[j];
            const uint32_t groups = (s_len[j] + 1023) / 1024;
            const uint32_t *mq = p.mask + (q0 + j) * p.groups * 32 + lane;
            for (uint32_t gr = 0; gr < groups; ++gr)
                pos += emit_words(__ldcs(mq + gr * 32), s_gb[j] + (uint64_t)gr * 1024, pos, p.out, p.cap, lane,
                                  s_off);
        }
    }
}

}  // namespace ckpt

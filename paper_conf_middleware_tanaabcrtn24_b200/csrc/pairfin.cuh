// pairfin.cuh -- the fused pair path's finishing work inside K1 (leaf kernel, PAIR "full" mode).
//
// Everything after the leaf hashes of the paper's path is done by the warps of the leaf
// kernel itself, as soon as its inputs exist, instead of by later kernels:
//
//  * interior levels (Alg. 1) of BOTH trees: the warp that completes the last
//    pair-task under a level-7 node (last-arriver counter) hashes that node's 7-level
//    subtree (128 children per run) in its shared-memory ring; the warp completing the
//    last such group under a level-14 node does the next 7 levels, and so on up to the
//    array root; the array roots then climb the top tree over all arrays (R15) the same
//    way.  Reading R13 makes every aligned group an exact subtree, so the nodes equal a
//    level-by-level build;
//  * the element test of the flagged chunks (verify): the warp that compares a
//    pair-task's leaf digests pushes one job per differing chunk onto a queue, and every
//    warp drains the queue before it draws its next leaf task (and after the last one,
//    until all pair-tasks are compared), so marking is spread over the whole grid and
//    overlaps the hashing instead of following it;
//  * ordered compaction: the warp that completes a tile (128 pair-tasks = 4096 chunks; the
//    pair-tasks' compares and the tile's marking jobs counted as work units) writes the
//    tile's flagged chunk ids in ascending order and each one's hit offset inside the tile.
//    One emit kernel (compare.cuh, pair_emit_kernel) then places chunk ids and element ids.
//
// Every hand-off is a release/acquire atomic on a counter that returns to zero in the
// launch (the last arriver resets it), so no buffer is cleared between launches.
#pragma once
#include <cstdint>

#include "hash.cuh"
#include "mark.cuh"
#include "mm32.cuh"

namespace ckpt {

constexpr int kMaxLv = 48;          // levels of one array tree (L < 2^47)
constexpr int kMaxSteps = 7;        // 7-level group steps (7 * 7 >= kMaxLv - 1)
constexpr int kGrpLog = 7;          // a group: 128 nodes of level 7j under one node of level 7j+7
constexpr int kTileTasks = 128;     // pair-tasks per tile (4096 chunks)
constexpr int kTileIds = kTileTasks * 32;
constexpr int kTileUnits = 33;      // work units per pair-task: its compare + up to 32 marked chunks
constexpr int kMaxTiles = 4096;     // tiles the emit kernel prefixes in shared memory

// Shape table of the two identically shaped trees (device, cached per shape by the host):
//   lvl [(m+1) * kMaxLv]    node index (from the tree base) of level k of array a; a = m is the
//                           top tree over the array roots
//   cb  [(m+1) * kMaxSteps] first group counter of step j (levels 7j -> 7j+7) of array a
//   nl  [m+1]               level-0 nodes of array a (the top tree: m)
struct TreeTab {
    const uint64_t *lvl;
    const uint32_t *cb;
    const uint64_t *nl;
};

struct PairParams {
    // ---- every pair mode ----
    unsigned int *ctr;            // [n_pair] pair-task arrival counters (0 between launches)
    uint64_t n_pair;              // pair-tasks (A's warp tasks)
    int m;                        // arrays per checkpoint
    uint8_t *flags;               // [L] 1 if the chunk's leaf digests differ, or null
    // ---- full mode (tmask != null) ----
    uint32_t *tmask;              // [n_pair] differing-chunk mask per pair-task
    uint64_t *tbase;              // [n_pair] global chunk id of the pair-task's chunk 0
    unsigned int *tctr;           // [n_tiles] work units arrived (0 between launches)
    uint32_t *tagg;               // [n_tiles] flagged chunks per tile
    uint64_t *thits;              // [n_tiles] differing elements per tile
    uint64_t *tids;               // [n_tiles * kTileIds] flagged chunk ids, ascending per tile
    uint32_t *tpos;               // [n_tiles * kTileIds] first hit of each listed chunk inside its tile
    TreeTab tab;
    uint4 *tree[2];               // node storage of run A's / run B's tree
    unsigned int *gctr;           // group counters (0 between launches)
    unsigned long long *q;        // [L] marking jobs: ((array << 44) | local chunk) + 1; 0 = empty
    unsigned long long *qs;       // [5] head, tail, pair-tasks compared, warps exited, jobs available
    unsigned long long *acc;      // [2] flagged chunks, differing elements (the emit kernel resets)
    uint32_t *cnt;                // [L] hits per flagged chunk (global chunk id)
    uint32_t *mask;               // [L * groups * 32] hit bits per flagged chunk (global chunk id)
    uint32_t groups;              // 32-word mask groups per chunk (1024 elements each)
    uint32_t per;                 // elements per chunk
    double eps;
};

__device__ __forceinline__ unsigned int atom_add_acq_rel(unsigned int *p, unsigned int v) {
    unsigned int old;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}
__device__ __forceinline__ unsigned long long atom_add_rel64(unsigned long long *p, unsigned long long v) {
    unsigned long long old;
    asm volatile("atom.release.gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}
__device__ __forceinline__ unsigned long long ld_acquire64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// levels of a tree over L >= 1 leaves: 1 + ceil(log2 L)  (n_{l+1} = ceil(n_l / 2), R13)
__device__ __forceinline__ int tree_height_dev(uint64_t L) {
    return L <= 1 ? 1 : 1 + (64 - __clzll((long long)(L - 1)));
}

// Levels lc+1 .. min(lc+7, H-1) of group g of array aa in BOTH trees: the children are the
// level-lc nodes [g*128, g*128 + cnt), the group's nodes at level lc+k start at g << (7-k).
// A node whose right child does not exist is promoted unchanged (R13).  `sm`: 512 nodes of
// warp-private shared memory (ping-pong, run r's nodes at [r*128 ..]).
__device__ __noinline__ void build_group(const PairParams &pr, int aa, int lc, int H, uint64_t g,
                                         uint32_t cnt, uint4 *sm, int lane) {
    const uint64_t *lvl = pr.tab.lvl + (uint64_t)aa * kMaxLv;
    uint4 *in = sm, *out = sm + 256;
    const uint64_t src = __ldg(lvl + lc) + (g << kGrpLog);
    for (uint32_t i = lane; i < 256; i += 32) {
        const uint32_t r = i >> 7, j = i & 127;
        if (j < cnt) in[i] = __ldcg(pr.tree[r] + src + j);
    }
    __syncwarp();
    uint32_t c = cnt;
    for (int k = 1; k <= kGrpLog && lc + k <= H - 1; ++k) {
        const uint32_t cn = (c + 1) >> 1;
        const uint64_t base = __ldg(lvl + lc + k) + (g << (kGrpLog - k));
        for (uint32_t i = lane; i < 2 * cn; i += 32) {
            const uint32_t r = i >= cn ? 1u : 0u, j = i - r * cn;
            uint4 x = in[r * 128 + 2 * j];
            if (2 * j + 1 < c) x = hash_children32(x, in[r * 128 + 2 * j + 1]);
            out[r * 128 + j] = x;
            pr.tree[r][base + j] = x;
        }
        __syncwarp();
        uint4 *t = in;
        in = out;
        out = t;
        c = cn;
    }
}

// One unit of array aa is complete: `first` -- pair-task u (leaves 32u .. 32u+31, both runs);
// otherwise node u of level lc (its whole subtree in both trees).  Arrive at the enclosing
// group's counter; the last arriver builds the group and climbs on.  An array root is copied
// to level 0 of the top tree (array index m) and climbs the top tree the same way.
__device__ __noinline__ void climb(const PairParams &pr, int aa, uint64_t u, bool first,
                                   uint4 *sm, int lane) {
    int lc = 0;
    for (;;) {
        const uint64_t L = __ldg(pr.tab.nl + aa);
        const int H = tree_height_dev(L);
        if (lc >= H - 1) {                       // node 0 of level H-1 is the root
            if (aa == pr.m) return;              // the checkpoint root: done
            const uint64_t top0 = __ldg(pr.tab.lvl + (uint64_t)pr.m * kMaxLv);
            if (lane < 2) {
                const uint4 root = __ldcg(pr.tree[lane] + __ldg(pr.tab.lvl + (uint64_t)aa * kMaxLv + H - 1));
                pr.tree[lane][top0 + aa] = root;
            }
            u = (uint64_t)aa;
            aa = pr.m;
            lc = 0;
            first = false;
            continue;
        }
        const uint64_t nlc = (L + (1ull << lc) - 1) >> lc;            // nodes of level lc
        const uint64_t g = first ? (u >> 2) : (u >> kGrpLog);
        const uint64_t left = nlc - (g << kGrpLog);
        const uint32_t cnt = (uint32_t)(left < 128 ? left : 128);
        const uint32_t target = first ? (cnt + 31) / 32 : cnt;
        unsigned int *c = pr.gctr + __ldg(pr.tab.cb + (uint64_t)aa * kMaxSteps + lc / kGrpLog) + g;
        __syncwarp();                            // this warp's node stores before the release
        unsigned int old = 0;
        if (lane == 0) {
            old = atom_add_acq_rel(c, 1u);
            if (old == target - 1) *c = 0u;      // last arriver: no other access this launch
        }
        old = __shfl_sync(0xffffffffu, old, 0);
        if (old != target - 1) return;
        __syncwarp();                            // lane 0's acquire, then every lane's loads
        build_group(pr, aa, lc, H, g, cnt, sm, lane);
        u = g;
        lc += kGrpLog;
        first = false;
    }
}

// The tile's ordered chunk list (ascending global chunk ids) and each listed chunk's first
// hit inside the tile; totals into tagg/thits and the launch accumulators.
__device__ __noinline__ void tile_finish(const PairParams &pr, uint64_t tile, int lane) {
    const uint64_t t0 = tile * kTileTasks;
    const uint64_t t1 = (t0 + kTileTasks) < pr.n_pair ? t0 + kTileTasks : pr.n_pair;
    uint64_t *dst = pr.tids + tile * kTileIds;
    uint32_t *dpos = pr.tpos + tile * kTileIds;
    uint32_t run = 0;
    uint64_t hrun = 0;
    for (uint64_t k = t0; k < t1; k += 32) {
        const uint64_t pt = k + lane;
        uint32_t m = 0;
        uint64_t b = 0;
        if (pt < t1) {
            m = __ldcg(pr.tmask + pt);
            b = __ldcg(reinterpret_cast<const unsigned long long *>(pr.tbase) + pt);
        }
        uint32_t hits = 0;
        for (uint32_t mm = m; mm; mm &= mm - 1) hits += __ldcg(pr.cnt + b + (__ffs(mm) - 1));
        uint32_t x = __popc(m), h = hits;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            const uint32_t z = __shfl_up_sync(0xffffffffu, h, o);
            if (lane >= o) { x += y; h += z; }
        }
        const uint32_t tot = __shfl_sync(0xffffffffu, x, 31);
        const uint32_t htot = __shfl_sync(0xffffffffu, h, 31);
        uint32_t pos = run + x - __popc(m);
        uint32_t hp = (uint32_t)hrun + h - hits;
        for (uint32_t mm = m; mm; mm &= mm - 1, ++pos) {
            const uint64_t gid = b + (uint64_t)(__ffs(mm) - 1);
            dst[pos] = gid;
            dpos[pos] = hp;
            hp += __ldcg(pr.cnt + gid);
        }
        run += tot;
        hrun += htot;
    }
    if (lane == 0) {
        pr.tagg[tile] = run;
        pr.thits[tile] = hrun;
        if (run) atomicAdd(pr.acc, (unsigned long long)run);
        if (hrun) atomicAdd(pr.acc + 1, (unsigned long long)hrun);
    }
}

// `units` work units of `tile` are done; the unit that completes the tile finishes it.
__device__ __forceinline__ void tile_arrive(const PairParams &pr, uint64_t tile, unsigned int units,
                                            int lane) {
    const uint64_t rest = pr.n_pair - tile * kTileTasks;
    const unsigned int target = kTileUnits * (unsigned int)(rest < kTileTasks ? rest : kTileTasks);
    __syncwarp();                                // this warp's stores before the release
    unsigned int old = 0;
    if (lane == 0) {
        old = atom_add_acq_rel(pr.tctr + tile, units);
        if (old + units == target) pr.tctr[tile] = 0u;
    }
    old = __shfl_sync(0xffffffffu, old, 0);
    if (old + units == target) {
        __syncwarp();
        tile_finish(pr, tile, lane);
    }
}

// Claim one marking job.  Pushers raise the tail, write their entries, then add to the
// "available" count; a claimer takes one unit of it with a fetch-and-add (no retry loop on
// a shared word: every claim is one round trip however many warps contend) and, on
// success, the next head slot, which is then guaranteed to be (or become) a written entry.
// A failed take (the count was not positive) is given back.  Returns the entry or 0.
__device__ __forceinline__ unsigned long long claim_job(const PairParams &pr, int lane) {
    unsigned long long e = 0;
    if (lane == 0) {
        long long *avail = reinterpret_cast<long long *>(pr.qs + 4);
        if (*reinterpret_cast<volatile long long *>(avail) > 0) {
            const long long before = (long long)atomicAdd(reinterpret_cast<unsigned long long *>(avail),
                                                          (unsigned long long)-1ll);
            if (before > 0) {
                const unsigned long long h = atomicAdd(pr.qs, 1ull);
                volatile unsigned long long *slot = pr.q + h;
                do { e = *slot; } while (e == 0ull);
                *slot = 0ull;                    // empty again for the next launch
            } else {
                atomicAdd(reinterpret_cast<unsigned long long *>(avail), 1ull);
            }
        }
    }
    return __shfl_sync(0xffffffffu, e, 0);
}

}  // namespace ckpt

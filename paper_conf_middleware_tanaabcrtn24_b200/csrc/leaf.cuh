// leaf.cuh -- K1: fused conservative rounding + block-chained Murmur3F leaf hash.
//
// Paper: Alg. 1 lines 3-12 and section 2.4.  The
// chain inside a chunk is serial (the digest of block b seeds block b+1,
// P:611-615), so the unit of parallelism is the chunk: every LANE owns one
// chunk's chain and a warp covers 32 consecutive chunks (a "task").
//
// Data movement: per warp, a ring of STAGES shared-memory slots, each slot
// holding a SEG-byte segment of each of the warp's 32 chunks, filled with
// 16-byte cp.async (LDGSTS, L2-only).  One cp.async warp instruction moves
// 512 contiguous-per-chunk bytes; rows are padded by 16 bytes so the
// per-lane 16-byte LDS of "my chunk, block b" is bank-conflict free.
// The ring is warp-private: only __syncwarp is needed, no CTA barriers.
//
// Grid: persistent, (SMs x resident CTAs); warps stride over tasks.
#pragma once
#include <cstdint>

#include "hash.cuh"
#include "mm32.cuh"

namespace ckpt {

struct LeafArray {            // one array of the checkpoint (device table)
    const uint8_t *data;      // 16-byte aligned
    uint64_t nbytes;
    uint64_t n_leaves;        // ceil(nbytes / C)
    uint64_t n_full;          // nbytes / C  (chunks of exactly C bytes)
    uint64_t task_begin;      // first global task id of this array
    uint4 *out;               // this array's leaf 0 in its tree's node storage
    uint64_t chunk_base;      // global chunk id of this array's chunk 0 in its tree
};

// Geometry (measured choices): 8-warp CTAs, 3 CTAs per SM (80
// registers), 128-byte segments per chunk per stage, a 2-slot ring, the f32 stage loop
// unrolled x2.
constexpr int kLeafWarps = 8;                  // warps per CTA
constexpr int kLeafMinBlocks = 3;              // resident CTAs per SM (register cap)
constexpr int kLeafUnroll = 2;                 // f32 stage-loop unroll
constexpr int kRows = 32;                      // chunks per warp task (one chain per lane)
constexpr int kSeg = 128;                      // bytes per chunk per stage
constexpr int kStages = 2;                     // ring depth
constexpr int kPitch = kSeg + 16;    // padded row
constexpr int kSlotBytes = kRows * kPitch;
constexpr int kWarpSmem = kStages * kSlotBytes;
constexpr int kLeafSmem = kLeafWarps * kWarpSmem + 16;   // + the two h*5+c addends

__device__ __forceinline__ void cp_async16(uint32_t smem, const void *gptr, uint32_t src_bytes) {
    asm volatile("cp.async.cg.shared.global.L2::128B [%0], [%1], 16, %2;\n" ::"r"(smem), "l"(gptr),
                 "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void cp_async16_full(uint32_t smem, const void *gptr) {
    asm volatile("cp.async.cg.shared.global.L2::128B [%0], [%1], 16;\n" ::"r"(smem), "l"(gptr)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}
__device__ __forceinline__ uint4 lds128(uint32_t addr) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];\n"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "r"(addr));
    return v;
}

// Exact hashed words of one 16-byte piece (raw bits in v): per-element
// fast/slow selection (generic path: ragged tasks and retries).
template <int DT, bool RAW>
__device__ __forceinline__ uint4 words_exact(uint4 v, const QuantParams &q) {
    uint4 w;
    if (RAW) {
        w = v;
    } else if (DT == 0) {
        w = make_uint4(word_f32(__uint_as_float(v.x), q), word_f32(__uint_as_float(v.y), q),
                       word_f32(__uint_as_float(v.z), q), word_f32(__uint_as_float(v.w), q));
    } else {
        const uint64_t k0 = word_f64(__hiloint2double((int)v.y, (int)v.x), q);
        const uint64_t k1 = word_f64(__hiloint2double((int)v.w, (int)v.z), q);
        w = make_uint4((uint32_t)k0, (uint32_t)(k0 >> 32), (uint32_t)k1, (uint32_t)(k1 >> 32));
    }
    return w;
}

// Hash one 16-byte block with exact words (canonical 16-byte hash blocks).
template <int DT, bool RAW>
__device__ __forceinline__ void chain_block_exact(U64p &h1, U64p &h2, uint4 v, const QuantParams &q) {
    const uint4 w = words_exact<DT, RAW>(v, q);
    mm3p_block16(h1, h2, U64p{w.x, w.y}, U64p{w.z, w.w}, q.m1, q.m2);
}

// Hash one 16-byte block with the branch-free fast rounding.  `ok` accumulates
// "every element so far was inside the fast range" (FSETP ... AND chains, no
// branch); a task whose warp saw any out-of-range element is redone exactly.
template <int DT, bool RAW>
__device__ __forceinline__ uint4 words_fast(uint4 v, const QuantParams &q, bool &ok, float &mx) {
    uint4 w;
    if (RAW) {
        w = v;
    } else if (DT == 0) {
        const float x0 = __uint_as_float(v.x), x1 = __uint_as_float(v.y);
        const float x2 = __uint_as_float(v.z), x3 = __uint_as_float(v.w);
        const double d0 = (double)x0, d1 = (double)x1, d2 = (double)x2, d3 = (double)x3;
        // running NaN-propagating max of |x| (two 3-input FMNMX3.NAN per block instead of
        // four FSETP); compared with r32 once per task
        asm("max.NaN.f32 %0, %1, %2, %3;" : "=f"(mx) : "f"(fabsf(x0)), "f"(fabsf(x1)), "f"(mx));
        asm("max.NaN.f32 %0, %1, %2, %3;" : "=f"(mx) : "f"(fabsf(x2)), "f"(fabsf(x3)), "f"(mx));
        // k mod 2^32 = low word of RD(x*inv + 1.5*2^52)   (hash.cuh)
        w.x = (uint32_t)__double2loint(__fma_rd(d0, q.inv, kMagic));
        w.y = (uint32_t)__double2loint(__fma_rd(d1, q.inv, kMagic));
        w.z = (uint32_t)__double2loint(__fma_rd(d2, q.inv, kMagic));
        w.w = (uint32_t)__double2loint(__fma_rd(d3, q.inv, kMagic));
    } else {
        const double x0 = __hiloint2double((int)v.y, (int)v.x);
        const double x1 = __hiloint2double((int)v.w, (int)v.z);
        ok = ok & (fabs(x0) < q.r64) & (fabs(x1) < q.r64);
        // k = bits(RD(x*inv + 1.5*2^52)) - bits(1.5*2^52); the low word of the magic is 0
        const double t0 = __fma_rd(x0, q.inv, kMagic);
        const double t1 = __fma_rd(x1, q.inv, kMagic);
        w.x = (uint32_t)__double2loint(t0);
        w.y = (uint32_t)__double2hiint(t0) - 0x43380000u;
        w.z = (uint32_t)__double2loint(t1);
        w.w = (uint32_t)__double2hiint(t1) - 0x43380000u;
    }
    return w;
}

template <int DT, bool RAW>
__device__ __forceinline__ void chain_block_fast(U64p &h1, U64p &h2, uint4 v, const QuantParams &q,
                                                 bool &ok, float &mx) {
    const uint4 w = words_fast<DT, RAW>(v, q, ok, mx);
    mm3p_block16<DT == 1>(h1, h2, U64p{w.x, w.y}, U64p{w.z, w.w}, q.m1, q.m2);
}

// Wide hash blocks (reading R23): a block of B = 16*hb16 bytes is
// one Murmur3F call, i.e. a body step per 16-byte piece and one finalisation
// (len = B) when the block is complete.  `left` counts the pieces still
// missing from the current block (uniform across the warp: no divergence).
__device__ __forceinline__ void wide_piece(U64p &h1, U64p &h2, uint4 w, const QuantParams &q,
                                           uint32_t &left, uint32_t hb16) {
    mm3p_body(h1, h2, U64p{w.x, w.y}, U64p{w.z, w.w}, q.m1, q.m2);
    if (--left == 0u) {
        mm3p_final(h1, h2, hb16 * 16u);
        left = hb16;
    }
}
// Short final block of `len` bytes (len in {4,8,12} for F32, 8 for F64),
// read straight from global memory (only the array's last chunk has one).
template <int DT, bool RAW>
__device__ __noinline__ void chain_tail(uint64_t &h1, uint64_t &h2, const uint8_t *p, uint32_t len,
                                        const QuantParams &q) {
    uint32_t w[4] = {0u, 0u, 0u, 0u};
    if (DT == 0) {
        for (uint32_t e = 0; e < len / 4; ++e) {
            const uint32_t bits = reinterpret_cast<const uint32_t *>(p)[e];
            w[e] = RAW ? bits : word_f32(__uint_as_float(bits), q);
        }
    } else {
        const uint64_t bits = reinterpret_cast<const uint64_t *>(p)[0];
        const uint64_t k = RAW ? bits : word_f64(__longlong_as_double((long long)bits), q);
        w[0] = (uint32_t)k;
        w[1] = (uint32_t)(k >> 32);
    }
    mm3_block_tail(h1, h2, (uint64_t)w[0] | ((uint64_t)w[1] << 32),
                   (uint64_t)w[2] | ((uint64_t)w[3] << 32), len);
}

// Wide-block variant of the chunk end: the <16-byte tail (if any) is mixed
// into the open block, then the open block (blen bytes, pieces + tail) is
// finalised with its own length, as Murmur3F does for a short key.
template <int DT, bool RAW>
__device__ __noinline__ void wide_end(uint64_t &h1, uint64_t &h2, const uint8_t *p, uint32_t tail,
                                      uint32_t blen, const QuantParams &q) {
    if (tail) {
        uint32_t w[4] = {0u, 0u, 0u, 0u};
        if (DT == 0) {
            for (uint32_t e = 0; e < tail / 4; ++e) {
                const uint32_t bits = reinterpret_cast<const uint32_t *>(p)[e];
                w[e] = RAW ? bits : word_f32(__uint_as_float(bits), q);
            }
        } else {
            const uint64_t bits = reinterpret_cast<const uint64_t *>(p)[0];
            const uint64_t k = RAW ? bits : word_f64(__longlong_as_double((long long)bits), q);
            w[0] = (uint32_t)k;
            w[1] = (uint32_t)(k >> 32);
        }
        uint64_t k1 = (uint64_t)w[0] | ((uint64_t)w[1] << 32);
        uint64_t k2 = (uint64_t)w[2] | ((uint64_t)w[3] << 32);
        if (tail > 8) {
            k2 *= kC2;
            k2 = rotl64(k2, 33);
            k2 *= kC1;
            h2 ^= k2;
        }
        k1 *= kC1;
        k1 = rotl64(k1, 31);
        k1 *= kC2;
        h1 ^= k1;
    }
    if (blen) mm3_final(h1, h2, blen);
}

constexpr int kLeafInline = 16;

// Fused pair mode: the table holds checkpoint A's m
// arrays then B's m arrays (identical shapes); warp task t < n_pair is A's
// task t, t >= n_pair is B's task t - n_pair (the usual batch order, so the
// warps in flight stream one checkpoint at a time).  Whichever of the two
// warps of a pair-task finishes second (a self-resetting atomicInc counter per
// pair-task) compares the 32 leaf digests and writes one flag byte per chunk:
// the diff at start level 0 happens inside K1.  (Marking the flagged chunks'
// elements here as well was measured slower than K4a: flagged chunks cluster,
// so the marking serialises in the few warps that own them.)
// Tile compaction (optional, tmask != null): pair-tasks are grouped in tiles
// of kTileTasks; the warp that completes a tile's last pair-task (a
// self-resetting acq_rel counter per tile) writes the tile's flagged chunk ids,
// ascending, to tids[tile * kTileTasks * 32 ..] and their number to tagg[tile].
// The ordered chunk list is then one gather pass (tile_gather_kernel) with no
// look-back: the digest compare, the flags AND their compaction happen in K1.
constexpr int kTileTasks = 128;                // pair-tasks per tile (4096 chunks)
struct PairParams {
    uint8_t *flags;               // [L] 1 if the chunk's leaf digests differ
    unsigned int *ctr;            // [n_pair] 0 between launches (atomicInc wraps 1 -> 0)
    uint64_t n_pair;              // pair-tasks (A's warp tasks)
    int m;                        // arrays per checkpoint
    uint32_t *tmask;              // [n_pair] differing-chunk mask per pair-task, or null
    uint64_t *tbase;              // [n_pair] global chunk id of the pair-task's chunk 0
    unsigned int *tctr;           // [n_tiles] 0 between launches
    uint32_t *tagg;               // [n_tiles] flagged chunks per tile
    uint64_t *tids;               // [n_tiles * kTileTasks * 32] tile-compacted chunk ids
};

// The tile's ordered chunk ids, by the warp that completed its last pair-task
// (after an acquire of every pair-task's release).
__device__ __noinline__ void tile_compact(const PairParams &pr, uint64_t tile, int lane) {
    const uint64_t t0 = tile * kTileTasks;
    const uint64_t t1 = (t0 + kTileTasks) < pr.n_pair ? t0 + kTileTasks : pr.n_pair;
    uint64_t *dst = pr.tids + t0 * 32;
    uint32_t run = 0;
    for (uint64_t k = t0; k < t1; k += 32) {
        const uint64_t pt = k + lane;
        uint32_t m = 0;
        uint64_t b = 0;
        if (pt < t1) {
            m = __ldcg(pr.tmask + pt);
            b = __ldcg(reinterpret_cast<const unsigned long long *>(pr.tbase) + pt);
        }
        uint32_t x = __popc(m);
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= o) x += y;
        }
        const uint32_t tot = __shfl_sync(0xffffffffu, x, 31);
        uint32_t pos = run + x - __popc(m);
        for (uint32_t mm = m; mm; mm &= mm - 1) dst[pos++] = b + (uint64_t)(__ffs(mm) - 1);
        run += tot;
    }
    if (lane == 0) pr.tagg[tile] = run;
}

struct LeafParams {
    const LeafArray *arrays;      // device table when n_arrays > kLeafInline
    LeafArray inl[kLeafInline];
    int n_arrays;
    uint64_t n_tasks;
    uint32_t chunk;
    QuantParams q;
    PairParams pr;
    // warps draw tasks in order from this counter (0 at launch; the final draw
    // resets it), so a warp held up elsewhere takes fewer tasks
    unsigned long long *ticket;
    // hash block in 16-byte pieces (WIDE kernels only): B = 16*hb16 <= C bytes;
    // B = C is one Murmur3F call per chunk
    uint32_t hb16;
};

__device__ __forceinline__ int find_array(const LeafArray *arr, int n_arrays, uint64_t task) {
    int lo = 0, hi = n_arrays - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (arr[mid].task_begin <= task) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// CB = chunk bytes if known at compile time (multiple of kSeg), else 0.
// A task is kRows = 32 consecutive chunks of one array; lane l owns the chain
// of chunk l of the task.
// WIDE: hash blocks of P.hb16 pieces (reading R23) instead of the paper's
// default 16-byte blocks.
// Chunks of >= 32 KB give few, long chains (often fewer than the GPU holds):
// those instantiations drop the 3-CTA register cap so ptxas keeps more of a
// chain's independent work in flight (measured +1-7% at 32 KB, +5-22% at 64 KB).
template <int DT, bool RAW, int CB, bool PAIR, bool WIDE>
__device__ __forceinline__ void leaf_body(const LeafParams &P) {
    pdl_enter();
    // small array tables travel in the kernel parameters (no H2D copy per build)
    const LeafArray *arrays = P.n_arrays <= kLeafInline ? P.inl : P.arrays;
    const int n_arrays = P.n_arrays;
    const uint64_t n_tasks = P.n_tasks;
    const uint32_t chunk_rt = P.chunk;
    QuantParams q = P.q;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const uint32_t C = CB ? (uint32_t)CB : chunk_rt;
    const uint32_t n_stages = (C + kSeg - 1) / kSeg;
    const uint32_t ring = (uint32_t)__cvta_generic_to_shared(smem + warp * kWarpSmem);
    constexpr int kPiecesPerChunk = kSeg / 16;            // 16-B pieces per chunk per stage
    constexpr int kChunksPerInstr = 32 / kPiecesPerChunk;  // rows covered by one warp instr
    constexpr int kLoads = kRows / kChunksPerInstr;        // cp.async per lane per stage
    const int my_q = lane / kPiecesPerChunk;                // first row I load
    const int my_sub = lane % kPiecesPerChunk;
    const uint32_t my_row = ring + (uint32_t)lane * kPitch;  // the row I hash
    // keep the h*5+c addends in vector registers (a uniform-register pair cannot be the
    // 64-bit addend of IMAD.WIDE; ptxas would split the add into IADD3 + IADD3.X)
    {
        uint64_t *cst = reinterpret_cast<uint64_t *>(smem + (blockDim.x >> 5) * kWarpSmem);
        if (threadIdx.x == 0) { cst[0] = q.m1; cst[1] = q.m2; }
        __syncthreads();
        q.m1 = *reinterpret_cast<volatile uint64_t *>(cst);
        q.m2 = *reinterpret_cast<volatile uint64_t *>(cst + 1);
    }

    // CTAs have kLeafWarps warps, or 1 when there are fewer tasks than resident warps (the
    // host then launches one CTA per task so that every SM gets the same number of chains)
    const uint32_t cta_warps = blockDim.x >> 5;
    const uint64_t n_warps_grid = (uint64_t)gridDim.x * cta_warps;
    auto draw = [&]() -> uint64_t {
        unsigned long long t = 0;
        if (lane == 0) {
            t = atomicAdd(P.ticket, 1ull);
            if (t == n_tasks + n_warps_grid - 1) *P.ticket = 0ull;   // the last draw of the launch
        }
        return __shfl_sync(0xffffffffu, t, 0);
    };
    for (uint64_t task = draw(); task < n_tasks; task = draw()) {
        const int a = find_array(arrays, n_arrays, task);
        const LeafArray A = arrays[a];
        const uint64_t c0 = (task - A.task_begin) * kRows;   // first local chunk of the task
        // wide blocks take the fast path only when they tile the chunk exactly
        const bool full_task = (C % kSeg == 0) && (c0 + kRows) <= A.n_full &&
                               (!WIDE || (C / 16) % P.hb16 == 0);
        U64p h1{0u, 0u}, h2{0u, 0u};
        bool done = false;

        if (full_task) {
            // ---------------- fast path: kRows full chunks ----------------
            const uint8_t *src = A.data + (c0 + my_q) * C + my_sub * 16;
            const uint32_t dst0 = ring + my_q * kPitch + my_sub * 16;
            auto issue = [&](const uint8_t *sp, uint32_t slot_off) {
#pragma unroll
                for (int i = 0; i < kLoads; ++i)
                    cp_async16_full(dst0 + slot_off + i * kChunksPerInstr * kPitch,
                                    sp + (uint64_t)i * kChunksPerInstr * C);
            };
            bool ok = true;
            float mx = 0.0f;
            const uint32_t hb16 = WIDE ? P.hb16 : 1u;
            uint32_t left = hb16;
#pragma unroll
            for (int s = 0; s < kStages - 1; ++s) {
                if ((uint32_t)s < n_stages) issue(src + s * kSeg, s * kSlotBytes);
                cp_async_commit();
            }
            src += (kStages - 1) * kSeg;
            uint32_t slot = 0u;                                   // slot of stage s
            uint32_t nslot = (kStages - 1) * kSlotBytes;          // slot of stage s+kStages-1
            // two stages per iteration (f32): the odd stage's cp.async addresses are the even
            // stage's + kSeg, an immediate offset (LDGSTS takes +-2 KB), so the 16 64-bit
            // address adds per stage are paid every other stage (86.5 -> 83.1 instructions
            // per 16-byte block; c2 pair launch 722 -> 706 us)
#pragma unroll (DT == 0 ? kLeafUnroll : 1)
            for (uint32_t s = 0; s < n_stages; ++s) {
                if (s + kStages - 1 < n_stages) issue(src, nslot);
                src += kSeg;
                nslot = (nslot == (kStages - 1) * kSlotBytes) ? 0u : nslot + kSlotBytes;
                cp_async_commit();
                cp_async_wait<kStages - 1>();
                __syncwarp();
                const uint32_t row = my_row + slot;
#pragma unroll
                for (int b = 0; b < kPiecesPerChunk; ++b) {
                    if constexpr (WIDE) {
                        const uint4 w = words_fast<DT, RAW>(lds128(row + b * 16), q, ok, mx);
                        wide_piece(h1, h2, w, q, left, hb16);
                    } else {
                        chain_block_fast<DT, RAW>(h1, h2, lds128(row + b * 16), q, ok, mx);
                    }
                }
                __syncwarp();
                slot = (slot == (kStages - 1) * kSlotBytes) ? 0u : slot + kSlotBytes;
            }
            cp_async_wait<0>();
            if (DT == 0 && !RAW) ok = ok & (mx < q.r32);     // NaN (propagated) fails
            done = __all_sync(0xffffffffu, ok);
        }
        if (!done) {
            // ------ exact path: ragged last task of an array, or a retry ------
            const uint64_t my_chunk = c0 + lane;
            uint64_t my_len = 0;
            if (my_chunk < A.n_leaves) {
                const uint64_t off = my_chunk * C;
                my_len = (A.nbytes - off) < C ? (A.nbytes - off) : C;
            }
            U64p e1{0u, 0u}, e2{0u, 0u};
            auto issue = [&](uint32_t s) {
                const uint32_t slot = ring + (s % kStages) * kSlotBytes;
#pragma unroll
                for (int i = 0; i < 32 / kChunksPerInstr; ++i) {
                    const int qq = my_q + i * kChunksPerInstr;
                    const uint64_t chunk = c0 + qq;
                    const uint64_t rel = (uint64_t)(s * kSeg + my_sub * 16);
                    const uint64_t off = chunk * C + rel;
                    uint32_t nb = 0;
                    if (chunk < A.n_leaves && off < A.nbytes && rel < C) {
                        uint64_t rem = A.nbytes - off;
                        const uint64_t crem = C - rel;
                        if (crem < rem) rem = crem;
                        // a piece shorter than 16 bytes is the chunk's Murmur3F tail,
                        // hashed from global memory (chain_tail / wide_end): not staged
                        nb = rem >= 16 ? 16u : 0u;
                    }
                    const uint8_t *sp = nb ? (A.data + off) : A.data;
                    cp_async16(slot + qq * kPitch + my_sub * 16, sp, nb);
                }
            };
#pragma unroll
            for (int s = 0; s < kStages - 1; ++s) {
                if ((uint32_t)s < n_stages) issue(s);
                cp_async_commit();
            }
            const uint64_t full_blocks = my_len / 16;
            // wide blocks: bytes in the open block of B = bbytes
            const uint32_t bbytes = WIDE ? P.hb16 * 16u : 16u;
            uint32_t blen = 0;
            for (uint32_t s = 0; s < n_stages; ++s) {
                if (s + kStages - 1 < n_stages) issue(s + kStages - 1);
                cp_async_commit();
                cp_async_wait<kStages - 1>();
                __syncwarp();
                const uint32_t row = my_row + (s % kStages) * kSlotBytes;
#pragma unroll
                for (int b = 0; b < kPiecesPerChunk; ++b) {
                    const uint64_t blk = (uint64_t)s * kPiecesPerChunk + b;
                    if (blk < full_blocks) {
                        if constexpr (WIDE) {
                            const uint4 w = words_exact<DT, RAW>(lds128(row + b * 16), q);
                            mm3p_body(e1, e2, U64p{w.x, w.y}, U64p{w.z, w.w}, q.m1, q.m2);
                            blen += 16u;
                            if (blen == bbytes) { mm3p_final(e1, e2, bbytes); blen = 0u; }
                        } else {
                            chain_block_exact<DT, RAW>(e1, e2, lds128(row + b * 16), q);
                        }
                    }
                }
                __syncwarp();
            }
            cp_async_wait<0>();
            __syncwarp();
            const uint32_t tail = (uint32_t)(my_len & 15);
            if (WIDE ? (tail | blen) != 0u : tail != 0u) {
                uint64_t t1 = ((uint64_t)e1.hi << 32) | e1.lo, t2 = ((uint64_t)e2.hi << 32) | e2.lo;
                if constexpr (WIDE)
                    wide_end<DT, RAW>(t1, t2, A.data + my_chunk * C + (my_len - tail), tail,
                                      blen + tail, q);
                else
                    chain_tail<DT, RAW>(t1, t2, A.data + my_chunk * C + (my_len - tail), tail, q);
                e1 = U64p{(uint32_t)t1, (uint32_t)(t1 >> 32)};
                e2 = U64p{(uint32_t)t2, (uint32_t)(t2 >> 32)};
            }
            h1 = e1;
            h2 = e2;
        }
        {
            const uint64_t c = c0 + lane;
            if (c < A.n_leaves) A.out[c] = make_uint4(h1.lo, h1.hi, h2.lo, h2.hi);
        }
        if constexpr (PAIR) {
            const int side = a >= P.pr.m ? 1 : 0;
            const uint64_t pt = task - (side ? P.pr.n_pair : 0);
            // publish my leaves, then count in; the second of the pair does the compare.
            // The warp barrier orders every lane's leaf stores before lane 0's
            // acq_rel atomic (release: cumulative over what the barrier made
            // visible to it; acquire: the other run's leaves, published by its
            // own release, are visible after the next barrier) -- no full fences.
            __syncwarp();
            unsigned int order = 0;
            if (lane == 0)
                asm volatile("atom.acq_rel.gpu.global.inc.u32 %0, [%1], 1;"
                             : "=r"(order) : "l"(&P.pr.ctr[pt]) : "memory");
            order = __shfl_sync(0xffffffffu, order, 0);
            if (order == 1) {
                __syncwarp();   // lane 0's acquire, then every lane's loads
                const LeafArray Pa = arrays[side ? a - P.pr.m : a + P.pr.m];   // the other run
                const uint64_t c = c0 + lane;
                bool differ = false;
                if (c < A.n_leaves) {
                    const uint4 o = __ldcg(Pa.out + c);
                    differ = (o.x != h1.lo) | (o.y != h1.hi) | (o.z != h2.lo) | (o.w != h2.hi);
                    P.pr.flags[A.chunk_base + c] = differ ? 1 : 0;
                }
                if (P.pr.tmask) {
                    // publish this pair-task's mask, then count it into its tile
                    const uint32_t m = __ballot_sync(0xffffffffu, differ);
                    const uint64_t tile = pt / kTileTasks;
                    const uint64_t rest = P.pr.n_pair - tile * kTileTasks;
                    const unsigned int in_tile = (unsigned int)(rest < kTileTasks ? rest : kTileTasks);
                    unsigned int done = 0;
                    if (lane == 0) {
                        P.pr.tmask[pt] = m;
                        P.pr.tbase[pt] = A.chunk_base + c0;
                        asm volatile("atom.acq_rel.gpu.global.inc.u32 %0, [%1], %2;"
                                     : "=r"(done) : "l"(P.pr.tctr + tile), "r"(in_tile - 1u) : "memory");
                    }
                    done = __shfl_sync(0xffffffffu, done, 0);
                    if (done == in_tile - 1u) {
                        __syncwarp();
                        tile_compact(P.pr, tile, lane);
                    }
                }
            }
        }
        __syncwarp();
    }
}

template <int DT, bool RAW, int CB, bool PAIR, bool WIDE = false>
__global__ void __launch_bounds__(kLeafWarps * 32, CB >= 32768 ? 1 : kLeafMinBlocks)
leaf_kernel(const __grid_constant__ LeafParams P) {
    leaf_body<DT, RAW, CB, PAIR, WIDE>(P);
}

// Fused f32 pair mode below 32 KB chunks: the same body capped at 72 registers instead of the
// 80 that three 8-warp CTAs per SM allow (same SASS instruction mix, different register
// assignment).  c2 leaf 685.5-685.9 vs 691.9-692.9 us over four alternating reps, c5 within
// noise; the f64 pair kernels stay at 80 (c3 at 512 B / 16 KiB chunks 0.8 % slower at 72).
// profiles/r2/follower_trials.md.
constexpr int kLeafPairRegs = 72;
constexpr uint32_t kLeafPairMaxChunk = 32768;
template <int DT, bool RAW, int CB, bool WIDE = false>
__global__ void __maxnreg__(kLeafPairRegs) leaf_pair_kernel(const __grid_constant__ LeafParams P) {
    leaf_body<DT, RAW, CB, true, WIDE>(P);
}

}  // namespace ckpt

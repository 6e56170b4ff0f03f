// leaf.cuh -- K1: fused conservative rounding + block-chained Murmur3F leaf hash.
//
// Paper: Alg. 1 lines 3-12 and section 2.4.  The
// chain inside a chunk is serial (the digest of block b seeds block b+1,
// P:611-615), so the unit of parallelism is the chunk: every LANE owns one
// chunk's chain and a warp covers 32 consecutive chunks (a "task").
//
// Fast path (task of 32 full chunks, chunk_bytes % 128 == 0): per warp a
// double-buffered ring of [32 chunks x 128 B] tiles in shared memory, each
// tile ONE TMA load (cp.async.bulk.tensor.2d over the array viewed as
// [n_chunks][chunk_bytes], 128-byte swizzle) issued by one lane and completed
// on an mbarrier.  Lane r reads its row's 16-byte block b at 16-byte unit
// b ^ (r & 7) (the swizzle), so the 8 lanes of a quarter-warp hit 8 distinct
// bank groups.  The per-block rounding is branch-free; `ok` accumulates an
// FSETP range test and a warp that saw an out-of-range element (NaN, inf,
// |x| >= r) redoes the task on the exact path.
//
// Exact path (an array's ragged last task, chunk sizes that are not a
// multiple of 128, retries): 16-byte cp.async with zero-fill into padded
// rows, exact per-element rounding, Murmur3F tail for a short last block.
//
// Grid: persistent, (SMs x resident CTAs); warps stride over tasks.
#pragma once
#include <cuda.h>
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
    const CUtensorMap *tmap;  // [n_full][C] byte view for the TMA fast path, or null
};

constexpr int kLeafWarps = 8;                  // warps per CTA
constexpr int kRows = 32;                      // chunks per warp task
// fast path (TMA)
constexpr int kSeg = 128;                      // bytes per chunk per stage (one swizzle row)
constexpr int kTileBytes = kRows * kSeg;       // 4 KiB, 1024-aligned slots
constexpr int kFastWarpSmem = 2 * kTileBytes;
// exact path (cp.async, padded rows)
constexpr int kSegX = 64;
constexpr int kPitchX = kSegX + 16;
constexpr int kSlotX = kRows * kPitchX;
constexpr int kExactWarpSmem = 2 * kSlotX;
constexpr int kWarpSmem = kFastWarpSmem > kExactWarpSmem ? kFastWarpSmem : kExactWarpSmem;
// dynamic smem: 1 KiB alignment slack + warp rings + 2 mbarriers per warp + the h*5+c addends
constexpr int kBarOff = kLeafWarps * kWarpSmem;
constexpr int kCstOff = kBarOff + kLeafWarps * 16;
constexpr int kLeafSmem = 1024 + kCstOff + 16;

__device__ __forceinline__ void cp_async16(uint32_t smem, const void *gptr, uint32_t src_bytes) {
    asm volatile("cp.async.cg.shared.global.L2::128B [%0], [%1], 16, %2;\n" ::"r"(smem), "l"(gptr),
                 "r"(src_bytes)
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

// --- mbarrier / TMA (sm_90+ PTX, used here on sm_100a) ---------------------
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}\n" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap *map, int x, int y,
                                            uint32_t bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3}], [%4];\n" ::"r"(dst),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(bar)
        : "memory");
}

// Hash one 16-byte block (raw bits in v), exact words for every input:
// per-element fast/slow selection (exact path).
template <int DT, bool RAW>
__device__ __forceinline__ void chain_block_exact(U64p &h1, U64p &h2, uint4 v, const QuantParams &q) {
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
    mm3p_block16(h1, h2, U64p{w.x, w.y}, U64p{w.z, w.w}, q.m1, q.m2);
}

// Hash one 16-byte block with the branch-free fast rounding.  `ok` accumulates
// "every element so far was inside the fast range" (FSETP ... AND chains).
template <int DT, bool RAW>
__device__ __forceinline__ void chain_block_fast(U64p &h1, U64p &h2, uint4 v, const QuantParams &q,
                                                 bool &ok) {
    uint4 w;
    if (RAW) {
        w = v;
    } else if (DT == 0) {
        const float x0 = __uint_as_float(v.x), x1 = __uint_as_float(v.y);
        const float x2 = __uint_as_float(v.z), x3 = __uint_as_float(v.w);
        const double d0 = (double)x0, d1 = (double)x1, d2 = (double)x2, d3 = (double)x3;
#ifdef CKPT_RANGE_F32
        ok = ok & (fabsf(x0) < q.r32) & (fabsf(x1) < q.r32) & (fabsf(x2) < q.r32) &
             (fabsf(x3) < q.r32);
#else
        // range test on the FP64 pipe (DSETP), which is otherwise nearly idle; the ALU
        // pipe is the leaf kernel's tightest (r32 <= r64, either bound keeps |x*inv| < 2^51)
        ok = ok & (fabs(d0) < q.r64) & (fabs(d1) < q.r64) & (fabs(d2) < q.r64) & (fabs(d3) < q.r64);
#endif
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
    mm3p_block16(h1, h2, U64p{w.x, w.y}, U64p{w.z, w.w}, q.m1, q.m2);
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

__device__ __forceinline__ int find_array(const LeafArray *arr, int n_arrays, uint64_t task) {
    int lo = 0, hi = n_arrays - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (arr[mid].task_begin <= task) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// Fast path over one task: chain states in h1/h2, returns whether every
// element was inside the fast range.  `bar` = this warp's two mbarriers,
// `phase` their parity bits (bit i for slot i), carried across tasks.
template <int DT, bool RAW, int CB>
__device__ __forceinline__ bool fast_task(const LeafArray &A, uint64_t c0, uint32_t C, uint32_t tiles,
                                          uint32_t bar, uint32_t &phase, int lane,
                                          uint32_t rd0, const QuantParams &q,
                                          U64p &h1, U64p &h2) {
    const uint32_t n_stages = CB ? (uint32_t)(CB / kSeg) : C / kSeg;
    const int y = (int)c0;
    auto issue = [&](uint32_t s, uint32_t slot) {
        if (lane == 0) {
            // order this warp's generic-proxy reads of the slot before the async-proxy refill
            asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
            mbar_expect_tx(bar + 8 * slot, kTileBytes);
            tma_load_2d(tiles + slot * kTileBytes, A.tmap, (int)(s * kSeg), y, bar + 8 * slot);
        }
    };
    bool ok = true;
    issue(0, 0);
    for (uint32_t s = 0; s < n_stages; s += 2) {
        // slot 0 holds stage s, slot 1 receives stage s+1
        if (s + 1 < n_stages) issue(s + 1, 1);
        mbar_wait(bar, phase & 1u);
        phase ^= 1u;
#pragma unroll
        for (int b = 0; b < kSeg / 16; ++b)
            chain_block_fast<DT, RAW>(h1, h2, lds128(rd0 ^ (uint32_t)(b << 4)), q, ok);
        __syncwarp();
        if (s + 1 >= n_stages) break;
        if (s + 2 < n_stages) issue(s + 2, 0);
        mbar_wait(bar + 8, (phase >> 1) & 1u);
        phase ^= 2u;
#pragma unroll
        for (int b = 0; b < kSeg / 16; ++b)
            chain_block_fast<DT, RAW>(h1, h2, lds128((rd0 ^ (uint32_t)(b << 4)) + kTileBytes), q, ok);
        __syncwarp();
    }
    return ok;
}

// Exact path over the 32 chunks starting at c0 of array A.
template <int DT, bool RAW>
__device__ __noinline__ void exact_task(const LeafArray &A, uint64_t c0, uint32_t C, uint32_t ring,
                                        int lane, const QuantParams &q, U64p &h1, U64p &h2) {
    constexpr int kPieces = kSegX / 16;          // 16-B pieces per chunk per stage
    constexpr int kPerInstr = 32 / kPieces;      // chunks covered by one warp instruction
    const int my_q = lane / kPieces, my_sub = lane % kPieces;
    const uint32_t my_row = ring + (uint32_t)lane * kPitchX;
    const uint32_t n_stages = (C + kSegX - 1) / kSegX;
    const uint64_t my_chunk = c0 + lane;
    uint64_t my_len = 0;
    if (my_chunk < A.n_leaves) {
        const uint64_t off = my_chunk * C;
        my_len = (A.nbytes - off) < C ? (A.nbytes - off) : C;
    }
    auto issue = [&](uint32_t s) {
        const uint32_t slot = ring + (s & 1u) * kSlotX;
#pragma unroll
        for (int i = 0; i < kRows / kPerInstr; ++i) {
            const int qq = my_q + i * kPerInstr;
            const uint64_t chunk = c0 + qq;
            const uint64_t rel = (uint64_t)(s * kSegX + my_sub * 16);
            const uint64_t off = chunk * C + rel;
            uint32_t nb = 0;
            if (chunk < A.n_leaves && off < A.nbytes && rel < C) {
                uint64_t rem = A.nbytes - off;
                const uint64_t crem = C - rel;
                if (crem < rem) rem = crem;
                nb = rem >= 16 ? 16u : (uint32_t)rem;
            }
            const uint8_t *sp = nb ? (A.data + off) : A.data;
            cp_async16(slot + qq * kPitchX + my_sub * 16, sp, nb);
        }
    };
    U64p e1{0u, 0u}, e2{0u, 0u};
    issue(0);
    cp_async_commit();
    const uint64_t full_blocks = my_len / 16;
    for (uint32_t s = 0; s < n_stages; ++s) {
        if (s + 1 < n_stages) issue(s + 1);
        cp_async_commit();
        cp_async_wait<1>();
        __syncwarp();
        const uint32_t row = my_row + (s & 1u) * kSlotX;
#pragma unroll
        for (int b = 0; b < kPieces; ++b) {
            const uint64_t blk = (uint64_t)s * kPieces + b;
            if (blk < full_blocks) chain_block_exact<DT, RAW>(e1, e2, lds128(row + b * 16), q);
        }
        __syncwarp();
    }
    cp_async_wait<0>();
    __syncwarp();
    const uint32_t tail = (uint32_t)(my_len & 15);
    if (tail) {
        uint64_t t1 = ((uint64_t)e1.hi << 32) | e1.lo, t2 = ((uint64_t)e2.hi << 32) | e2.lo;
        chain_tail<DT, RAW>(t1, t2, A.data + my_chunk * C + (my_len - tail), tail, q);
        e1 = U64p{(uint32_t)t1, (uint32_t)(t1 >> 32)};
        e2 = U64p{(uint32_t)t2, (uint32_t)(t2 >> 32)};
    }
    h1 = e1;
    h2 = e2;
}

// CB = chunk bytes if known at compile time (multiple of kSeg), else 0.
template <int DT, bool RAW, int CB>
#ifndef CKPT_LEAF_MINB
#define CKPT_LEAF_MINB 2
#endif
__global__ void __launch_bounds__(kLeafWarps * 32, CKPT_LEAF_MINB)
leaf_kernel(const LeafArray *__restrict__ arrays, int n_arrays, uint64_t n_tasks, uint32_t chunk_rt,
            QuantParams q) {
    extern __shared__ __align__(16) uint8_t smem_raw[];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const uint32_t C = CB ? (uint32_t)CB : chunk_rt;
    const uint32_t raw = (uint32_t)__cvta_generic_to_shared(smem_raw);
    const uint32_t base = (raw + 1023u) & ~1023u;              // 1 KiB aligned (128B swizzle)
    uint8_t *smem = smem_raw + (base - raw);
    const uint32_t ring = base + warp * kWarpSmem;
    const uint32_t bar = base + kBarOff + warp * 16;
    {
        uint64_t *cst = reinterpret_cast<uint64_t *>(smem + kCstOff);
        if (threadIdx.x == 0) { cst[0] = q.m1; cst[1] = q.m2; }
        if (lane == 0) {
            mbar_init(bar, 1);
            mbar_init(bar + 8, 1);
            asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        }
        __syncthreads();
        // keep the h*5+c addends in vector registers (a uniform-register pair cannot be the
        // 64-bit addend of IMAD.WIDE; ptxas would split the add)
        q.m1 = *reinterpret_cast<volatile uint64_t *>(cst);
        q.m2 = *reinterpret_cast<volatile uint64_t *>(cst + 1);
    }
    // my row's 16-byte blocks in a swizzled tile: unit b of row r sits at b ^ (r & 7)
    // (ring + lane*128 has zero bits 4..6, so the swizzled address of block b is rd0 ^ (b << 4))
    const uint32_t rd0 = ring + (uint32_t)lane * kSeg + ((uint32_t)(lane & 7) << 4);
    uint32_t phase = 0u;

    for (uint64_t task = (uint64_t)blockIdx.x * kLeafWarps + warp; task < n_tasks;
         task += (uint64_t)gridDim.x * kLeafWarps) {
        const int a = find_array(arrays, n_arrays, task);
        const LeafArray &A = arrays[a];
        const uint64_t c0 = (task - A.task_begin) * kRows;   // first local chunk of the task
        const bool fast = A.tmap != nullptr && (C % kSeg == 0) && (c0 + kRows) <= A.n_full;
        U64p h1{0u, 0u}, h2{0u, 0u};
        bool done = false;
        if (fast) {
            const bool ok = fast_task<DT, RAW, CB>(A, c0, C, ring, bar, phase, lane, rd0, q, h1, h2);
            done = __all_sync(0xffffffffu, ok);
        }
        if (!done) exact_task<DT, RAW>(A, c0, C, ring, lane, q, h1, h2);
        const uint64_t c = c0 + lane;
        if (c < A.n_leaves) A.out[c] = make_uint4(h1.lo, h1.hi, h2.lo, h2.hi);
        __syncwarp();
    }
}

}  // namespace ckpt

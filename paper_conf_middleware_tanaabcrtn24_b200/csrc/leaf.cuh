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

namespace ckpt {

struct LeafArray {            // one array of the checkpoint (device table)
    const uint8_t *data;      // 16-byte aligned
    uint64_t nbytes;
    uint64_t n_leaves;        // ceil(nbytes / C)
    uint64_t n_full;          // nbytes / C  (chunks of exactly C bytes)
    uint64_t task_begin;      // first global task id of this array
    uint64_t leaf_off;        // node index of this array's leaf 0
};

constexpr int kLeafWarps = 8;        // warps per CTA
constexpr int kSeg = 64;             // bytes per chunk per stage
constexpr int kStages = 4;           // ring depth
constexpr int kPitch = kSeg + 16;    // padded row
constexpr int kSlotBytes = 32 * kPitch;
constexpr int kWarpSmem = kStages * kSlotBytes;
constexpr int kLeafSmem = kLeafWarps * kWarpSmem;

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

// Hash one 16-byte block of input (as 4 u32 lanes of raw bits) into (h1,h2).
template <int DT, bool RAW>
__device__ __forceinline__ void chain_block(uint64_t &h1, uint64_t &h2, uint4 v, const QuantParams &q) {
    uint64_t k1, k2;
    if (RAW) {
        k1 = (uint64_t)v.x | ((uint64_t)v.y << 32);
        k2 = (uint64_t)v.z | ((uint64_t)v.w << 32);
    } else if (DT == 0) {
        const float x0 = __uint_as_float(v.x), x1 = __uint_as_float(v.y);
        const float x2 = __uint_as_float(v.z), x3 = __uint_as_float(v.w);
        const bool fast = (fabsf(x0) < q.r32) & (fabsf(x1) < q.r32) & (fabsf(x2) < q.r32) &
                          (fabsf(x3) < q.r32);
        uint32_t w0, w1, w2, w3;
        if (fast) {
            w0 = (uint32_t)__double2loint(__fma_rd((double)x0, q.inv, kMagic));
            w1 = (uint32_t)__double2loint(__fma_rd((double)x1, q.inv, kMagic));
            w2 = (uint32_t)__double2loint(__fma_rd((double)x2, q.inv, kMagic));
            w3 = (uint32_t)__double2loint(__fma_rd((double)x3, q.inv, kMagic));
        } else {
            w0 = word_f32(x0, q);
            w1 = word_f32(x1, q);
            w2 = word_f32(x2, q);
            w3 = word_f32(x3, q);
        }
        k1 = (uint64_t)w0 | ((uint64_t)w1 << 32);
        k2 = (uint64_t)w2 | ((uint64_t)w3 << 32);
    } else {
        const double x0 = __hiloint2double((int)v.y, (int)v.x);
        const double x1 = __hiloint2double((int)v.w, (int)v.z);
        const bool fast = (fabs(x0) < q.r64) & (fabs(x1) < q.r64);
        if (fast) {
            k1 = (uint64_t)__double_as_longlong(__fma_rd(x0, q.inv, kMagic)) - kMagicBits;
            k2 = (uint64_t)__double_as_longlong(__fma_rd(x1, q.inv, kMagic)) - kMagicBits;
        } else {
            k1 = word_f64(x0, q);
            k2 = word_f64(x1, q);
        }
    }
    mm3_block16(h1, h2, k1, k2);
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

// CB = chunk bytes if known at compile time (multiple of kSeg), else 0.
template <int DT, bool RAW, int CB>
__global__ void __launch_bounds__(kLeafWarps * 32)
leaf_kernel(const LeafArray *__restrict__ arrays, int n_arrays, uint64_t n_tasks, uint32_t chunk_rt,
            QuantParams q, uint4 *__restrict__ nodes) {
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const uint32_t C = CB ? (uint32_t)CB : chunk_rt;
    const uint32_t n_stages = (C + kSeg - 1) / kSeg;
    const uint32_t ring = (uint32_t)__cvta_generic_to_shared(smem + warp * kWarpSmem);
    constexpr int kPiecesPerChunk = kSeg / 16;           // 16-B pieces per chunk per stage
    constexpr int kChunksPerInstr = 32 / kPiecesPerChunk; // chunks covered by one warp instr
    const int my_q = lane / kPiecesPerChunk;               // chunk (within 8-group) I load
    const int my_sub = lane % kPiecesPerChunk;
    const uint32_t my_row = ring + (uint32_t)lane * kPitch;  // the row I hash

    for (uint64_t task = (uint64_t)blockIdx.x * kLeafWarps + warp; task < n_tasks;
         task += (uint64_t)gridDim.x * kLeafWarps) {
        const int a = find_array(arrays, n_arrays, task);
        const LeafArray A = arrays[a];
        const uint64_t c0 = (task - A.task_begin) * 32;      // first local chunk of the task
        const uint8_t *base = A.data + c0 * C;
        const uint64_t my_chunk = c0 + lane;
        const bool full_task = (C % kSeg == 0) && (c0 + 32) <= A.n_full;
        // bytes of my (hashed) chunk
        uint64_t my_len = 0;
        if (my_chunk < A.n_leaves) {
            const uint64_t off = my_chunk * C;
            my_len = (A.nbytes - off) < C ? (A.nbytes - off) : C;
        }
        uint64_t h1 = 0, h2 = 0;

        if (full_task) {
            // ---------------- fast path: 32 full chunks ----------------
            auto issue = [&](uint32_t s) {
                const uint32_t slot = ring + (s % kStages) * kSlotBytes;
                const uint8_t *src = base + (uint64_t)my_q * C + s * kSeg + my_sub * 16;
                const uint32_t dst = slot + my_q * kPitch + my_sub * 16;
#pragma unroll
                for (int i = 0; i < 32 / kChunksPerInstr; ++i)
                    cp_async16_full(dst + i * kChunksPerInstr * kPitch,
                                    src + (uint64_t)i * kChunksPerInstr * C);
            };
#pragma unroll
            for (int s = 0; s < kStages - 1; ++s) {
                if ((uint32_t)s < n_stages) issue(s);
                cp_async_commit();
            }
            for (uint32_t s = 0; s < n_stages; ++s) {
                if (s + kStages - 1 < n_stages) issue(s + kStages - 1);
                cp_async_commit();
                cp_async_wait<kStages - 1>();
                __syncwarp();
                const uint32_t row = my_row + (s % kStages) * kSlotBytes;
#pragma unroll
                for (int b = 0; b < kPiecesPerChunk; ++b)
                    chain_block<DT, RAW>(h1, h2, lds128(row + b * 16), q);
                __syncwarp();
            }
        } else {
            // ------------- ragged path: the array's last task -------------
            auto issue = [&](uint32_t s) {
                const uint32_t slot = ring + (s % kStages) * kSlotBytes;
#pragma unroll
                for (int i = 0; i < 32 / kChunksPerInstr; ++i) {
                    const int qq = my_q + i * kChunksPerInstr;
                    const uint64_t chunk = c0 + qq;
                    const uint64_t off = chunk * C + s * kSeg + my_sub * 16;
                    uint32_t nb = 0;
                    const uint64_t chunk_end_rel = (uint64_t)(s * kSeg + my_sub * 16);
                    if (chunk < A.n_leaves && off < A.nbytes && chunk_end_rel < C) {
                        uint64_t rem = A.nbytes - off;
                        uint64_t crem = C - chunk_end_rel;
                        if (crem < rem) rem = crem;
                        nb = rem >= 16 ? 16u : (uint32_t)rem;
                    }
                    const uint8_t *src = nb ? (A.data + off) : A.data;
                    cp_async16(slot + qq * kPitch + my_sub * 16, src, nb);
                }
            };
#pragma unroll
            for (int s = 0; s < kStages - 1; ++s) {
                if ((uint32_t)s < n_stages) issue(s);
                cp_async_commit();
            }
            const uint64_t full_blocks = my_len / 16;
            for (uint32_t s = 0; s < n_stages; ++s) {
                if (s + kStages - 1 < n_stages) issue(s + kStages - 1);
                cp_async_commit();
                cp_async_wait<kStages - 1>();
                __syncwarp();
                const uint32_t row = my_row + (s % kStages) * kSlotBytes;
#pragma unroll
                for (int b = 0; b < kPiecesPerChunk; ++b) {
                    const uint64_t blk = (uint64_t)s * kPiecesPerChunk + b;
                    if (blk < full_blocks) chain_block<DT, RAW>(h1, h2, lds128(row + b * 16), q);
                }
                __syncwarp();
            }
            const uint32_t tail = (uint32_t)(my_len & 15);
            if (tail) chain_tail<DT, RAW>(h1, h2, A.data + my_chunk * C + (my_len - tail), tail, q);
        }
        cp_async_wait<0>();
        if (my_chunk < A.n_leaves) nodes[A.leaf_off + my_chunk] = digest(h1, h2);
        __syncwarp();
    }
}

}  // namespace ckpt

// mark.cuh -- the element test of step a5 (verify) over one chunk:
// hit bits of fabs((double)a_i - (double)b_i) > eps (reading R9), written as a
// bitmask, plus the hit count.  Used by K4a (verify_mark_kernel) and by the
// fused pair leaf kernel (leaf.cuh, PAIR mode).
#pragma once
#include <cstdint>

namespace ckpt {

constexpr int kVerifyBatch = 4;   // warp iterations whose loads are issued together

// Bits of |a-b| > eps (computed in double, reading R9) for the VEC elements
// of one 16-byte vector pair.
template <int DT>
__device__ __forceinline__ uint32_t diff_vec(uint4 va, uint4 vb, double eps) {
    uint32_t m = 0;
    if (DT == 0) {
        m |= (fabs((double)__uint_as_float(va.x) - (double)__uint_as_float(vb.x)) > eps) ? 1u : 0u;
        m |= (fabs((double)__uint_as_float(va.y) - (double)__uint_as_float(vb.y)) > eps) ? 2u : 0u;
        m |= (fabs((double)__uint_as_float(va.z) - (double)__uint_as_float(vb.z)) > eps) ? 4u : 0u;
        m |= (fabs((double)__uint_as_float(va.w) - (double)__uint_as_float(vb.w)) > eps) ? 8u : 0u;
    } else {
        const double a0 = __hiloint2double((int)va.y, (int)va.x), b0 = __hiloint2double((int)vb.y, (int)vb.x);
        const double a1 = __hiloint2double((int)va.w, (int)va.z), b1 = __hiloint2double((int)vb.w, (int)vb.z);
        m |= (fabs(a0 - b0) > eps) ? 1u : 0u;
        m |= (fabs(a1 - b1) > eps) ? 2u : 0u;
    }
    return m;
}

// Scalar tail: elements e.. of a vector that crosses the chunk end.
template <int DT>
__device__ __forceinline__ uint32_t diff_tail(const uint8_t *pa, const uint8_t *pb, uint64_t e,
                                              uint64_t len, double eps) {
    constexpr int VEC = DT == 0 ? 4 : 2;
    uint32_t m = 0;
    for (int v = 0; v < VEC; ++v) {
        if (e + v >= len) break;
        double x, y;
        if (DT == 0) {
            x = (double)reinterpret_cast<const float *>(pa)[e + v];
            y = (double)reinterpret_cast<const float *>(pb)[e + v];
        } else {
            x = reinterpret_cast<const double *>(pa)[e + v];
            y = reinterpret_cast<const double *>(pb)[e + v];
        }
        if (fabs(x - y) > eps) m |= 1u << v;
    }
    return m;
}

// One warp marks one chunk of len elements at pa / pb (16-byte aligned):
// writes ceil(len/1024) groups of 32 mask words to mask[g*32 + lane] (word w
// holds elements 32w..32w+31, element-contiguous) and returns the hit count
// (the same value in every lane).
template <int DT, int BATCH = kVerifyBatch>
__device__ __forceinline__ uint32_t mark_chunk(const uint8_t *pa, const uint8_t *pb, uint64_t len,
                                               double eps, uint32_t *mask, int lane) {
    constexpr unsigned kAll = 0xffffffffu;
    constexpr int VEC = DT == 0 ? 4 : 2;
    constexpr int kStep = 32 * VEC;            // elements per warp iteration
    constexpr int IPG = 32 / VEC;              // warp iterations per group of 32 mask words
    constexpr int LPW = 32 / VEC;              // lanes contributing to one mask word
    const uint4 *qa = reinterpret_cast<const uint4 *>(pa);
    const uint4 *qb = reinterpret_cast<const uint4 *>(pb);
    uint32_t *mq = mask + lane;
    uint32_t cnt = 0, word = 0;
    int it = 0;
    for (uint64_t base = 0; base < len; base += (uint64_t)BATCH * kStep) {
        uint4 va[BATCH], vb[BATCH];
#pragma unroll
        for (int u = 0; u < BATCH; ++u) {
            const uint64_t e = base + (uint64_t)u * kStep + (uint64_t)lane * VEC;
            if (e + VEC <= len) {
                va[u] = __ldcs(qa + e / VEC);
                vb[u] = __ldcs(qb + e / VEC);
            }
        }
#pragma unroll
        for (int u = 0; u < BATCH; ++u) {
            const uint64_t e0 = base + (uint64_t)u * kStep;
            if (e0 >= len) break;                          // warp-uniform
            const uint64_t e = e0 + (uint64_t)lane * VEC;
            uint32_t m = 0;
            if (e + VEC <= len) m = diff_vec<DT>(va[u], vb[u], eps);
            else if (e < len) m = diff_tail<DT>(pa, pb, e, len, eps);
            cnt += __popc(m);
            // transpose to element-contiguous words: word k of this iteration
            // (elements k*32.. of its 32*VEC) is gathered from LPW lanes and
            // lands in lane (it % IPG) * VEC + k
            uint32_t x = m << (VEC * (lane % LPW));
#pragma unroll
            for (int o = 1; o < LPW; o <<= 1) x |= __shfl_xor_sync(kAll, x, o);
            const uint32_t y = __shfl_sync(kAll, x, (lane % VEC) * LPW);
            if (lane / VEC == it % IPG) word = y;
            if (++it % IPG == 0) { __stcs(mq, word); mq += 32; word = 0; }
        }
    }
    if (it % IPG) __stcs(mq, word);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(kAll, cnt, o);
    return cnt;
}

}  // namespace ckpt

// hash.cuh -- device Murmur3F and error-bounded rounding for sm_100a.
//
// Murmur3F: the 128-bit "Murmur3F" of P:588-594 (SMHasher footnote P:652) is
// MurmurHash3_x64_128 (reading R1).  The leaf chain of P:607-615 / Alg. 1
// P:501-511 calls it once per 16-byte block with the previous digest as the
// full 128-bit starting state (R2, R4).  Interior nodes hash the 32-byte
// concatenation of the two children with seed 0 (Alg. 1, R14).
//
// Rounding (R5-R9): k(x) = clamp(floor(x * inv), int64), inv =
// RN(1/eps), exact product, NaN -> 0.  Two independent evaluations:
//   * fast path (|x| < R, so |x*inv| < 2^51): one DFMA in round-down mode,
//     t = RD(x*inv + 1.5*2^52).  In the binade [2^52, 2^53) the doubles are
//     exactly the integers, so t = floor(x*inv) + 1.5*2^52 and the low
//     mantissa bits of t are k in two's complement (offset 2^51, which is
//     0 mod 2^32).  F32 word = low 32 bits of t; F64 word = bits(t) -
//     bits(1.5*2^52).
//   * slow path (NaN, inf, huge |x|): exact 128-bit integer product of the
//     two significands, shifted with floor semantics and clamped.
#pragma once
#include <cstdint>

namespace ckpt {

// Programmatic dependent launch: every kernel of the library is launched with
// programmatic stream serialisation, waits for its stream predecessor to
// complete (griddepcontrol.wait: full completion and memory visibility) before
// touching memory, and lets its own successor be scheduled right away, so the
// successor's launch and CTA rasterisation overlap this kernel's tail.  Both
// instructions are no-ops for a kernel launched without the attribute.
__device__ __forceinline__ void pdl_enter() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

constexpr uint64_t kC1 = 0x87c37b91114253d5ull;
constexpr uint64_t kC2 = 0x4cf5ad432745937full;
constexpr uint64_t kF1 = 0xff51afd7ed558ccdull;
constexpr uint64_t kF2 = 0xc4ceb9fe1a85ec53ull;

__device__ __forceinline__ uint64_t rotl64(uint64_t x, int r) {
    return (x << r) | (x >> (64 - r));
}

__device__ __forceinline__ uint64_t fmix64(uint64_t k) {
    k ^= k >> 33;
    k *= kF1;
    k ^= k >> 33;
    k *= kF2;
    k ^= k >> 33;
    return k;
}

// Murmur3F body step for one full 16-byte block (k1 = bytes 0..7 LE, k2 = 8..15).
__device__ __forceinline__ void mm3_body(uint64_t &h1, uint64_t &h2, uint64_t k1, uint64_t k2) {
    k1 *= kC1;
    k1 = rotl64(k1, 31);
    k1 *= kC2;
    h1 ^= k1;
    h1 = rotl64(h1, 27);
    h1 += h2;
    h1 = h1 * 5 + 0x52dce729ull;
    k2 *= kC2;
    k2 = rotl64(k2, 33);
    k2 *= kC1;
    h2 ^= k2;
    h2 = rotl64(h2, 31);
    h2 += h1;
    h2 = h2 * 5 + 0x38495ab5ull;
}

// Murmur3F finalisation with total byte length `len`.
__device__ __forceinline__ void mm3_final(uint64_t &h1, uint64_t &h2, uint64_t len) {
    h1 ^= len;
    h2 ^= len;
    h1 += h2;
    h2 += h1;
    h1 = fmix64(h1);
    h2 = fmix64(h2);
    h1 += h2;
    h2 += h1;
}

// One chained block: a complete Murmur3F call on 16 bytes from state (h1,h2).
__device__ __forceinline__ void mm3_block16(uint64_t &h1, uint64_t &h2, uint64_t k1, uint64_t k2) {
    mm3_body(h1, h2, k1, k2);
    mm3_final(h1, h2, 16);
}

// One chained short block of `len` in [1,15] bytes; k1/k2 zero-padded LE words.
__device__ __forceinline__ void mm3_block_tail(uint64_t &h1, uint64_t &h2, uint64_t k1, uint64_t k2,
                                               uint32_t len) {
    if (len > 8) {
        k2 *= kC2;
        k2 = rotl64(k2, 33);
        k2 *= kC1;
        h2 ^= k2;
    }
    k1 *= kC1;
    k1 = rotl64(k1, 31);
    k1 *= kC2;
    h1 ^= k1;
    mm3_final(h1, h2, len);
}

// Interior node: Murmur3F(left || right, 32 bytes, seed 0).
__device__ __forceinline__ uint4 hash_children(uint4 l, uint4 r) {
    uint64_t h1 = 0, h2 = 0;
    mm3_body(h1, h2, (uint64_t)l.x | ((uint64_t)l.y << 32), (uint64_t)l.z | ((uint64_t)l.w << 32));
    mm3_body(h1, h2, (uint64_t)r.x | ((uint64_t)r.y << 32), (uint64_t)r.z | ((uint64_t)r.w << 32));
    mm3_final(h1, h2, 32);
    return make_uint4((uint32_t)h1, (uint32_t)(h1 >> 32), (uint32_t)h2, (uint32_t)(h2 >> 32));
}

__device__ __forceinline__ uint4 digest(uint64_t h1, uint64_t h2) {
    return make_uint4((uint32_t)h1, (uint32_t)(h1 >> 32), (uint32_t)h2, (uint32_t)(h2 >> 32));
}

__device__ __forceinline__ bool digest_ne(uint4 a, uint4 b) {
    return ((a.x ^ b.x) | (a.y ^ b.y) | (a.z ^ b.z) | (a.w ^ b.w)) != 0u;
}

// ---------------------------------------------------------------------------
// rounding
// ---------------------------------------------------------------------------

struct QuantParams {
    double inv;        // RN(1/eps)
    double r64;        // fast path iff |x| < r64 (f64 input)
    uint64_t inv_m;    // inv = inv_m * 2^inv_e exactly
    int32_t inv_e;
    float r32;         // fast path iff |x| < r32 (f32 input)
    uint64_t m1, m2;   // Murmur3F body constants 0x52dce729 / 0x38495ab5 (see mm32.cuh)
};

constexpr double kMagic = 6755399441055744.0;            // 1.5 * 2^52
constexpr uint64_t kMagicBits = 0x4338000000000000ull;

// Exact k(x) by integer arithmetic (slow path; any double x).
__device__ __noinline__ int64_t quant_k_exact(double x, uint64_t mi, int ei) {
    const uint64_t bits = (uint64_t)__double_as_longlong(x);
    uint32_t ex = (uint32_t)(bits >> 52) & 0x7ffu;
    const bool neg = (bits >> 63) != 0;
    uint64_t mx = bits & 0xFFFFFFFFFFFFFull;
    if (ex == 0x7ffu) {
        if (mx != 0) return 0;                                 // NaN
        return neg ? INT64_MIN : INT64_MAX;                    // +-inf
    }
    if (ex == 0) {
        if (mx == 0) return 0;                                 // +-0
        ex = 1;                                                // subnormal
    } else {
        mx |= 1ull << 52;
    }
    const int e = (int)ex - 1075 + ei;                         // |x*inv| = mx*mi*2^e
    const uint64_t lo = mx * mi;
    const uint64_t hi = __umul64hi(mx, mi);
    uint64_t q, qhi;
    bool frac;
    if (e >= 0) {
        if (hi != 0 || e >= 63 || (lo >> (63 - e)) != 0) return neg ? INT64_MIN : INT64_MAX;
        q = lo << e;
        return neg ? -(int64_t)q : (int64_t)q;
    }
    const int s = -e;
    if (s >= 128) {
        q = 0;
        qhi = 0;
        frac = (hi | lo) != 0;
    } else if (s >= 64) {
        q = (s == 64) ? hi : (hi >> (s - 64));
        qhi = 0;
        frac = lo != 0 || (s > 64 && (hi << (128 - s)) != 0);
    } else {
        q = (lo >> s) | (hi << (64 - s));
        qhi = hi >> s;
        frac = (lo << (64 - s)) != 0;
    }
    if (!neg) {
        if (qhi != 0 || (q >> 63) != 0) return INT64_MAX;
        return (int64_t)q;
    }
    // floor(-V) = -ceil(V)
    const uint64_t c = q + (frac ? 1u : 0u);
    const uint64_t chi = qhi + (c < q ? 1u : 0u);
    if (chi != 0 || c > (1ull << 63)) return INT64_MIN;
    return (int64_t)(0ull - c);
}

// F32 word of one element (low 32 bits of k).
__device__ __forceinline__ uint32_t word_f32(float x, const QuantParams &q) {
    if (fabsf(x) < q.r32) {
        const double t = __fma_rd((double)x, q.inv, kMagic);
        return (uint32_t)__double2loint(t);
    }
    return (uint32_t)(uint64_t)quant_k_exact((double)x, q.inv_m, q.inv_e);
}

// F64 word of one element (k).
__device__ __forceinline__ uint64_t word_f64(double x, const QuantParams &q) {
    if (fabs(x) < q.r64) {
        const double t = __fma_rd(x, q.inv, kMagic);
        return (uint64_t)__double_as_longlong(t) - kMagicBits;
    }
    return (uint64_t)quant_k_exact(x, q.inv_m, q.inv_e);
}

}  // namespace ckpt

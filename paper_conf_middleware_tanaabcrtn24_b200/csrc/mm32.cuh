// mm32.cuh -- Murmur3F chained block step written on 32-bit register halves.
//
// Same function as mm3_block16 in hash.cuh (MurmurHash3_x64_128 on one
// 16-byte block from state (h1,h2), finalised with len = 16; P:607-615,
// R2-R4), re-expressed so that ptxas emits the minimum instruction stream
// on sm_100a and splits it across the two integer pipes:
//   * 64-bit x constant -> IMAD.WIDE.U32 + 2 x IMAD (fma pipe, 3 instr),
//   * k ^= k >> 33      -> lo ^= hi >> 1 (SHF + LOP3),
//   * rotl64 by r       -> two funnel shifts (SHF.L.W) on swapped halves,
//   * h*5 + c           -> IMAD.WIDE.U32 with a 64-bit addend + one IMAD.
// The leaf kernel is issue-bound, so every instruction
// of this step is throughput.
#pragma once
#include <cstdint>

namespace ckpt {

struct U64p {      // a 64-bit value as two 32-bit registers
    uint32_t lo, hi;
};

__device__ __forceinline__ U64p mulc(U64p a, uint32_t cl, uint32_t ch) {
    // (a * C) mod 2^64 = lo(a.lo*cl) | (hi(a.lo*cl) + a.lo*ch + a.hi*cl) << 32
    U64p r;
    uint32_t h;
    asm("{\n\t"
        ".reg .u64 p;\n\t"
        "mul.wide.u32 p, %2, %4;\n\t"
        "mov.b64 {%0, %1}, p;\n\t"
        "}"
        : "=r"(r.lo), "=r"(h)
        : "r"(a.lo), "r"(a.hi), "r"(cl));
    asm("mad.lo.u32 %0, %1, %2, %0;" : "+r"(h) : "r"(a.lo), "r"(ch));
    asm("mad.lo.u32 %0, %1, %2, %0;" : "+r"(h) : "r"(a.hi), "r"(cl));
    r.hi = h;
    return r;
}

// rotl64 by r in (0, 32)
template <int R>
__device__ __forceinline__ U64p rotl_lt32(U64p a) {
    U64p r;
    r.hi = __funnelshift_l(a.lo, a.hi, R);   // (hi << R) | (lo >> (32-R))
    r.lo = __funnelshift_l(a.hi, a.lo, R);   // (lo << R) | (hi >> (32-R))
    return r;
}

// rotl64 by r in (32, 64): swap halves, then rotate by r - 32
template <int R>
__device__ __forceinline__ U64p rotl_gt32(U64p a) {
    U64p s{a.hi, a.lo};
    return rotl_lt32<R - 32>(s);
}

__device__ __forceinline__ U64p xor64(U64p a, U64p b) { return U64p{a.lo ^ b.lo, a.hi ^ b.hi}; }

__device__ __forceinline__ U64p add64(U64p a, U64p b) {
    U64p r;
    asm("add.cc.u32 %0, %2, %4;\n\taddc.u32 %1, %3, %5;"
        : "=r"(r.lo), "=r"(r.hi)
        : "r"(a.lo), "r"(a.hi), "r"(b.lo), "r"(b.hi));
    return r;
}

// h*5 + c: lo*5 + c as one IMAD.WIDE.U32 (64-bit addend folded), then hi*5 + that
// product's high word as ONE IMAD: 2 instructions (81.1 vs 83.1 per block with the plain
// 64-bit product; an inline-asm mad.wide with an immediate multiplier was split by ptxas
// into IMAD.WIDE + IADD3 + IMAD.X, measured 1.8% slower)
__device__ __forceinline__ U64p mul5_add(U64p h, uint64_t c) {
    const uint64_t x = (uint64_t)h.lo * 5u + c;
    return U64p{(uint32_t)x, h.hi * 5u + (uint32_t)(x >> 32)};
}

__device__ __forceinline__ U64p xorshift33(U64p k) { return U64p{k.lo ^ (k.hi >> 1), k.hi}; }

__device__ __forceinline__ U64p fmix64p(U64p k) {
    k = xorshift33(k);
    k = mulc(k, 0xed558ccdu, 0xff51afd7u);
    k = xorshift33(k);
    k = mulc(k, 0x1a85ec53u, 0xc4ceb9feu);
    k = xorshift33(k);
    return k;
}

// Murmur3F body, key half: k1 = rotl(k1*c1, 31)*c2, k2 = rotl(k2*c2, 33)*c1.  It does
// not depend on the state, so a chain can mix the keys of later blocks ahead.
__device__ __forceinline__ void mm3p_kmix(U64p &k1, U64p &k2) {
    // c1 = 0x87c37b91114253d5, c2 = 0x4cf5ad432745937f
    k1 = mulc(k1, 0x114253d5u, 0x87c37b91u);
    k1 = rotl_lt32<31>(k1);
    k1 = mulc(k1, 0x2745937fu, 0x4cf5ad43u);
    k2 = mulc(k2, 0x2745937fu, 0x4cf5ad43u);
    k2 = rotl_gt32<33>(k2);
    k2 = mulc(k2, 0x114253d5u, 0x87c37b91u);
}

// Murmur3F body, state half, with mixed keys.
__device__ __forceinline__ void mm3p_hstep(U64p &h1, U64p &h2, U64p k1, U64p k2, uint64_t m1,
                                           uint64_t m2) {
    h1 = xor64(h1, k1);
    h1 = rotl_lt32<27>(h1);
    h1 = add64(h1, h2);
    h1 = mul5_add(h1, m1);   // m1 = 0x52dce729
    h2 = xor64(h2, k2);
    h2 = rotl_lt32<31>(h2);
    h2 = add64(h2, h1);
    h2 = mul5_add(h2, m2);   // m2 = 0x38495ab5
}

// Murmur3F body step for one full 16-byte block.
__device__ __forceinline__ void mm3p_body(U64p &h1, U64p &h2, U64p k1, U64p k2, uint64_t m1,
                                          uint64_t m2) {
    mm3p_kmix(k1, k2);
    mm3p_hstep(h1, h2, k1, k2, m1, m2);
}

// Murmur3F finalisation for a total length `len` < 2^32.
__device__ __forceinline__ void mm3p_final(U64p &h1, U64p &h2, uint32_t len) {
    h1.lo ^= len;
    h2.lo ^= len;
    h1 = add64(h1, h2);
    h2 = add64(h2, h1);
    h1 = fmix64p(h1);
    h2 = fmix64p(h2);
    h1 = add64(h1, h2);
    h2 = add64(h2, h1);
}

// a + b + b: "h1 += h2; h2 += h1" as two independent adds, the second a 3-input
// add that ptxas emits as IADD3 + IADD3.X (ALU pipe) instead of IADD3 + IMAD.X
__device__ __forceinline__ U64p add64_abb(U64p a, U64p b) {
    U64p r;
    asm("add.cc.u32 %0, %2, %4;\n\taddc.u32 %1, %3, %5;\n\t"
        "add.cc.u32 %0, %0, %4;\n\taddc.u32 %1, %1, %5;"
        : "=&r"(r.lo), "=&r"(r.hi)
        : "r"(a.lo), "r"(a.hi), "r"(b.lo), "r"(b.hi));
    return r;
}

// The same finalisation with the second add of each pair as add64_abb: the same
// instruction count, two carries moved from the FMA-heavy pipe to the ALU.  Used by
// the f64 leaf chain, whose FMA-heavy pipe binds (f64 pair launch 711 -> 663 us);
// the f32 chain is faster with the default (675 vs 692 us).
__device__ __forceinline__ void mm3p_final_alu(U64p &h1, U64p &h2, uint32_t len) {
    h1.lo ^= len;
    h2.lo ^= len;
    {
        const U64p a = add64(h1, h2), b = add64_abb(h1, h2);
        h1 = a;
        h2 = b;
    }
    h1 = fmix64p(h1);
    h2 = fmix64p(h2);
    {
        const U64p a = add64(h1, h2), b = add64_abb(h1, h2);
        h1 = a;
        h2 = b;
    }
}

// One chained 16-byte block: (h1,h2) <- Murmur3F(k1||k2, len 16, state (h1,h2)).
template <bool ALU_ADDS = false>
__device__ __forceinline__ void mm3p_block16(U64p &h1, U64p &h2, U64p k1, U64p k2, uint64_t m1,
                                             uint64_t m2) {
    mm3p_body(h1, h2, k1, k2, m1, m2);
    if (ALU_ADDS) mm3p_final_alu(h1, h2, 16u);
    else mm3p_final(h1, h2, 16u);
}

// Interior node: Murmur3F(left || right, 32 bytes, seed 0)  (Alg. 1, R14).
__device__ __forceinline__ uint4 hash_children32(uint4 l, uint4 r) {
    U64p h1{0u, 0u}, h2{0u, 0u};
    mm3p_body(h1, h2, U64p{l.x, l.y}, U64p{l.z, l.w}, 0x52dce729ull, 0x38495ab5ull);
    mm3p_body(h1, h2, U64p{r.x, r.y}, U64p{r.z, r.w}, 0x52dce729ull, 0x38495ab5ull);
    mm3p_final(h1, h2, 32u);
    return make_uint4(h1.lo, h1.hi, h2.lo, h2.hi);
}

}  // namespace ckpt

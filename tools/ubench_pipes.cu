// Instruction-throughput microbenchmark for the ops the leaf hash is made of.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench_pipes tools/ubench_pipes.cu
// Each thread runs 8 independent dependency chains of one op for N iterations;
// reported: warp-instructions per clock per SM (4.0 = one per SMSP per clock).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define N_ITER 4096

#define CHAIN8(stmt)                                                                    \
    stmt(a0) stmt(a1) stmt(a2) stmt(a3) stmt(a4) stmt(a5) stmt(a6) stmt(a7)

template <int OP>
__global__ void k(uint32_t *out, uint32_t seed) {
    uint32_t a0 = seed + threadIdx.x, a1 = a0 * 3, a2 = a0 * 5, a3 = a0 * 7, a4 = a0 * 11,
             a5 = a0 * 13, a6 = a0 * 17, a7 = a0 * 19;
    uint32_t b = seed ^ 0x9e3779b9u, c = seed * 0x85ebca6bu;
    double d0 = a0, d1 = a1, d2 = a2, d3 = a3, d4 = a4, d5 = a5, d6 = a6, d7 = a7;
    float f0 = a0, f1 = a1, f2 = a2, f3 = a3, f4 = a4, f5 = a5, f6 = a6, f7 = a7;
#pragma unroll 1
    for (int i = 0; i < N_ITER; ++i) {
        if (OP == 0) {   // IMAD reg,reg,reg
#define S(x) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x) : "r"(b), "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 1) {   // IMAD reg,imm,reg
#define S(x) asm volatile("mad.lo.u32 %0, %0, 0x2745937f, %1;" : "+r"(x) : "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 2) {   // IMAD.WIDE.U32 (two outputs)
#define S(x) asm volatile("{.reg .u64 p; mul.wide.u32 p, %0, 0x2745937f; cvt.u32.u64 %0, p;}" : "+r"(x));
            CHAIN8(S)
#undef S
        } else if (OP == 3) {   // IMAD.HI.U32
#define S(x) asm volatile("mad.hi.u32 %0, %0, 0x2745937f, %1;" : "+r"(x) : "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 4) {   // SHF.L.W
#define S(x) asm volatile("shf.l.wrap.b32 %0, %0, %1, 13;" : "+r"(x) : "r"(b));
            CHAIN8(S)
#undef S
        } else if (OP == 5) {   // LOP3
#define S(x) asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x) : "r"(b), "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 6) {   // IADD3
#define S(x) asm volatile("add.u32 %0, %0, %1;" : "+r"(x) : "r"(b));
            CHAIN8(S)
#undef S
        } else if (OP == 7) {   // IMAD + LOP3 interleaved (pipe overlap)
#define S(x) asm volatile("mad.lo.u32 %0, %0, 0x2745937f, %1;\n\tlop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x) : "r"(b), "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 8) {   // F2F.F64.F32
#define S(x) { double t; asm volatile("cvt.f64.f32 %0, %1;" : "=d"(t) : "f"(f##x)); d##x += t; }
            S(0) S(1) S(2) S(3) S(4) S(5) S(6) S(7)
#undef S
        } else if (OP == 9) {   // DFMA.RM
#define S(x) asm volatile("fma.rm.f64 %0, %0, %1, 0d4338000000000000;" : "+d"(d##x) : "d"(1.0000001));
            S(0) S(1) S(2) S(3) S(4) S(5) S(6) S(7)
#undef S
        } else if (OP == 10) {  // IADD3 with carry pair (64-bit add)
#define S(x) asm volatile("add.cc.u32 %0, %0, %1; addc.u32 %1, %1, %0;" : "+r"(x), "+r"(b));
            CHAIN8(S)
#undef S
        } else if (OP == 11) {  // FSETP chained
#define S(x) { uint32_t t; asm volatile("{.reg .pred q; setp.lt.f32 q, %1, %2; selp.u32 %0, 1, 0, q;}" : "=r"(t) : "f"(f##x), "f"(3.0f)); a##x += t; f##x += 1.0f; }
            S(0) S(1) S(2) S(3) S(4) S(5) S(6) S(7)
#undef S
        } else if (OP == 12) {  // IMAD.WIDE with 64-bit register addend
#define S(x) asm volatile("{.reg .u64 p, q; mov.b64 q, {%1, %2}; mad.wide.u32 p, %0, 5, q; cvt.u32.u64 %0, p;}" : "+r"(x) : "r"(b), "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 14) {  // 64-bit add as IMAD.WIDE.U32 x*1 + pair (FMA pipe)
#define S(x) asm volatile("{.reg .u64 p, q; mov.b64 q, {%1, %2}; mad.wide.u32 p, %0, 1, q; mov.b64 {%0, %1}, p;}" : "+r"(x), "+r"(b) : "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 15) {  // mad.lo x*2^k + y (IMAD.SHL-style shift-add)
#define S(x) asm volatile("mad.lo.u32 %0, %0, 32, %1;" : "+r"(x) : "r"(b));
            CHAIN8(S)
#undef S
        } else if (OP == 16) {  // PRMT
#define S(x) asm volatile("prmt.b32 %0, %0, %1, 0x3210;" : "+r"(x) : "r"(b));
            CHAIN8(S)
#undef S
        } else if (OP == 17) {  // 2 IMAD imm + 1 LOP3
#define S(x) asm volatile("mad.lo.u32 %0, %0, 0x2745937f, %1;\n\tmad.lo.u32 %0, %0, 0x114253d5, %2;\n\tlop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x) : "r"(b), "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 18) {  // SHF + IMAD imm
#define S(x) asm volatile("shf.l.wrap.b32 %0, %0, %1, 13;\n\tmad.lo.u32 %0, %0, 0x2745937f, %1;" : "+r"(x) : "r"(b));
            CHAIN8(S)
#undef S
        } else if (OP == 19) {  // IMAD.WIDE imm + LOP3
#define S(x) asm volatile("{.reg .u64 p; mul.wide.u32 p, %0, 0x2745937f; cvt.u32.u64 %0, p;}\n\tlop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x) : "r"(b), "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 20) {  // 3 IMAD imm + 1 LOP3 + 1 SHF
#define S(x) asm volatile("mad.lo.u32 %0, %0, 0x2745937f, %1;\n\tmad.lo.u32 %0, %0, 0x114253d5, %2;\n\tlop3.b32 %0, %0, %1, %2, 0x96;\n\tmad.lo.u32 %0, %0, 0x1a85ec53, %2;\n\tshf.l.wrap.b32 %0, %0, %1, 13;" : "+r"(x) : "r"(b), "r"(c));
            CHAIN8(S)
#undef S
        } else if (OP == 21) {  // IMAD.MOV-free 2-reg IMAD imm x*imm (no addend)
#define S(x) asm volatile("mul.lo.u32 %0, %0, 0x2745937f;" : "+r"(x));
            CHAIN8(S)
#undef S
        } else if (OP == 13) {  // FFMA (reference)
#define S(x) asm volatile("fma.rn.f32 %0, %0, 1.0001, 0.5;" : "+f"(f##x));
            S(0) S(1) S(2) S(3) S(4) S(5) S(6) S(7)
#undef S
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] =
        a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 + (uint32_t)(d0 + d1 + d2 + d3 + d4 + d5 + d6 + d7) +
        (uint32_t)(f0 + f1 + f2 + f3 + f4 + f5 + f6 + f7) + b;
}

template <int OP>
void run(const char *name, int sms, uint32_t *out, int instr_per_chain) {
    dim3 grid(sms * 4), block(512);   // 64 warps / SM
    k<OP><<<grid, block>>>(out, 1);
    cudaDeviceSynchronize();
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) k<OP><<<grid, block>>>(out, r);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    int clk_khz;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    double warp_instr = 5.0 * grid.x * (block.x / 32) * (double)N_ITER * 8 * instr_per_chain;
    double cycles = ms * 1e-3 * clk_khz * 1e3;   // at the nominal max clock
    printf("%-28s %6.3f warp-instr/clk/SM  (%.3f ms)\n", name, warp_instr / cycles / sms, ms / 5);
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    uint32_t *out;
    cudaMalloc(&out, sms * 4 * 512 * 4);
    run<0>("IMAD r,r,r", sms, out, 1);
    run<1>("IMAD r,imm,r", sms, out, 1);
    run<2>("IMAD.WIDE.U32 imm", sms, out, 1);
    run<12>("IMAD.WIDE.U32 +pair", sms, out, 1);
    run<3>("IMAD.HI.U32", sms, out, 1);
    run<4>("SHF.L.W", sms, out, 1);
    run<5>("LOP3", sms, out, 1);
    run<6>("IADD3", sms, out, 1);
    run<10>("IADD3 cc+X (2 instr)", sms, out, 2);
    run<7>("IMAD+LOP3 (2 instr)", sms, out, 2);
    run<11>("FSETP+SEL (2 instr)", sms, out, 2);
    run<8>("F2F.F64.F32 + DADD (2)", sms, out, 2);
    run<9>("DFMA.RM", sms, out, 1);
    run<13>("FFMA", sms, out, 1);
    run<14>("IMAD.WIDE x*1+pair (64b add)", sms, out, 1);
    run<15>("IMAD x*32+y", sms, out, 1);
    run<16>("PRMT", sms, out, 1);
    run<17>("2 IMAD imm + LOP3 (3)", sms, out, 3);
    run<18>("SHF + IMAD imm (2)", sms, out, 2);
    run<19>("IMAD.WIDE imm + LOP3 (2)", sms, out, 2);
    run<20>("3 IMADi+LOP3+SHF (5)", sms, out, 5);
    run<21>("IMUL imm", sms, out, 1);
    return 0;
}

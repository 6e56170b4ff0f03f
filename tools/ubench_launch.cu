// Fixed per-kernel costs on B200: empty kernel, dependent global round trips,
// griddepcontrol, fences, large parameter blocks.  Events around N back-to-back launches.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ubench_launch tools/ubench_launch.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

struct Big { uint64_t w[560]; };   // ~4.5 KB of parameters

__global__ void k_empty() {}
__global__ void k_pdl() { asm volatile("griddepcontrol.wait;" ::: "memory"); asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__global__ void k_chain(uint64_t *p, int n) {   // n dependent L2 round trips (one thread)
    if (threadIdx.x) return;
    uint64_t i = 0;
    for (int k = 0; k < n; ++k) i = __ldcg((const unsigned long long *)p + i);
    p[1000] = i;
}
__global__ void k_big(const __grid_constant__ Big b, uint64_t *out) { if (threadIdx.x == 0) out[0] = b.w[threadIdx.x + 5]; }
__global__ void k_bigaddr(const __grid_constant__ Big b, uint64_t *out, int j) {
    const uint64_t *q = b.w;   // address taken: generic loads from the param block
    if (threadIdx.x == 0) out[0] = q[j] + q[j + 7];
}
__global__ void k_fence(unsigned *t) { __syncthreads(); if (threadIdx.x == 0) { __threadfence(); atomicAdd(t, 1u); } }
__global__ void k_acqrel(unsigned *t) {
    __syncthreads();
    if (threadIdx.x == 0) { unsigned r; asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(r) : "l"(t) : "memory"); }
}

template <class F>
void timeit(const char *name, F launch, int reps = 200) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int i = 0; i < 10; ++i) launch();
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    for (int i = 0; i < reps; ++i) launch();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("%-36s %8.2f us per launch\n", name, ms * 1e3 / reps);
}

int main() {
    uint64_t *p; cudaMalloc(&p, 1 << 20); cudaMemset(p, 0, 1 << 20);
    unsigned *t; cudaMalloc(&t, 64);
    Big b{}; 
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cudaLaunchConfig_t cfg{}; cfg.gridDim = dim3(1); cfg.blockDim = dim3(256); cfg.attrs = at; cfg.numAttrs = 1;
    timeit("empty 1 CTA", [&] { k_empty<<<1, 256>>>(); });
    timeit("empty 148 CTAs", [&] { k_empty<<<148, 256>>>(); });
    timeit("empty 592 CTAs", [&] { k_empty<<<592, 256>>>(); });
    timeit("pdl-wait 1 CTA (PDL launch)", [&] { cudaLaunchKernelEx(&cfg, k_pdl); });
    timeit("pdl-wait 1 CTA (plain launch)", [&] { k_pdl<<<1, 256>>>(); });
    for (int n : {1, 10, 40})  {
        char nm[64]; snprintf(nm, 64, "chain of %d L2 loads", n);
        timeit(nm, [&] { k_chain<<<1, 32>>>(p, n); });
    }
    timeit("4.5 KB params", [&] { k_big<<<1, 256>>>(b, p); });
    timeit("4.5 KB params, address taken", [&] { k_bigaddr<<<1, 256>>>(b, p, 3); });
    timeit("threadfence + atomic, 148 CTAs", [&] { k_fence<<<148, 256>>>(t); });
    timeit("acq_rel atomic, 148 CTAs", [&] { k_acqrel<<<148, 256>>>(t); });
    return 0;
}

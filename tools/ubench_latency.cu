// Latency microbenchmark: dependent global loads (pointer chase), atomics, fences,
// and empty-kernel launch cost, timed with CUDA events.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ubench_latency tools/ubench_latency.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void chase(const uint64_t *p, int hops, uint64_t *out) {
    uint64_t i = 0;
    for (int h = 0; h < hops; ++h) i = __ldcg(p + i);
    if (threadIdx.x == 0) *out = i;
}
__global__ void atomics(unsigned long long *c, int n, uint64_t *out) {
    unsigned long long v = 0;
    for (int h = 0; h < n; ++h) v = atomicAdd(c, 1ull + (v & 0));
    if (threadIdx.x == 0) *out = v;
}
__global__ void fences(uint64_t *x, int n) {
    for (int h = 0; h < n; ++h) { x[threadIdx.x] = h; __threadfence(); }
}
__global__ void empty() {}

int main() {
    const int N = 1 << 20;
    uint64_t *p, *out;
    cudaMalloc(&p, N * 8);
    cudaMalloc(&out, 64);
    uint64_t *h = new uint64_t[N];
    // random cycle with 4 KiB stride-ish hops
    for (int i = 0; i < N; ++i) h[i] = (uint64_t)((i * 2654435761ull + 4099) % N);
    cudaMemcpy(p, h, N * 8, cudaMemcpyHostToDevice);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float ms;
    for (int hops : {1, 10, 100, 1000}) {
        chase<<<1, 32>>>(p, hops, out);
        cudaDeviceSynchronize();
        cudaEventRecord(a);
        for (int r = 0; r < 10; ++r) chase<<<1, 32>>>(p, hops, out);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("chase hops=%5d  %8.2f us/kernel  -> %6.1f ns/hop\n", hops, ms * 100, ms * 1e5 / hops);
    }
    for (int n : {1, 100, 1000}) {
        atomics<<<1, 32>>>((unsigned long long *)out, n, out + 1);
        cudaDeviceSynchronize();
        cudaEventRecord(a);
        for (int r = 0; r < 10; ++r) atomics<<<1, 32>>>((unsigned long long *)out, n, out + 1);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("atomics n=%5d  %8.2f us/kernel  -> %6.1f ns/op\n", n, ms * 100, ms * 1e5 / n);
    }
    for (int n : {1, 100}) {
        fences<<<1, 256>>>(p, n);
        cudaDeviceSynchronize();
        cudaEventRecord(a);
        for (int r = 0; r < 10; ++r) fences<<<1, 256>>>(p, n);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("fence  n=%5d  %8.2f us/kernel  -> %6.1f ns/op\n", n, ms * 100, ms * 1e5 / n);
    }
    for (int grid : {1, 148, 1184}) {
        empty<<<grid, 256>>>();
        cudaDeviceSynchronize();
        cudaEventRecord(a);
        for (int r = 0; r < 100; ++r) empty<<<grid, 256>>>();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("empty kernel grid=%5d: %6.2f us each (back-to-back)\n", grid, ms * 10);
        // single kernel bracketed by events
        cudaEventRecord(a);
        empty<<<grid, 256>>>();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("   single bracketed: %6.2f us\n", ms * 1e3);
    }
    return 0;
}

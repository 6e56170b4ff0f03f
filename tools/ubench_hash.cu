// Microbenchmark: latency of one interior-node hash (hash_children32) on sm_100a.
//   (1) one warp, a dependent chain of N hashes: cycles per hash (pure latency);
//   (2) one warp, 4 independent chains interleaved: cycles per hash (ILP 4);
//   (3) 32 warps on one SM, one chain each: throughput.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_middleware_tanaabcrtn24_b200/csrc tools/ubench_hash.cu -o tools/ubench_hash
#include <cstdio>
#include <cstdint>
#include "mm32.cuh"

using namespace ckpt;

template <int ILP>
__global__ void chain(uint4 *out, int n, long long *cyc) {
    uint4 x[ILP], y;
    for (int i = 0; i < ILP; ++i) x[i] = make_uint4(threadIdx.x + i, 1u, 2u, 3u);
    y = make_uint4(7u, threadIdx.x, 9u, 10u);
    __syncthreads();
    const long long t0 = clock64();
    for (int k = 0; k < n; ++k) {
#pragma unroll
        for (int i = 0; i < ILP; ++i) x[i] = hash_children32(x[i], y);
    }
    const long long t1 = clock64();
    uint4 r = x[0];
    for (int i = 1; i < ILP; ++i) r.x ^= x[i].x;
    out[blockIdx.x * blockDim.x + threadIdx.x] = r;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
    uint4 *out;
    long long *cyc, h[64];
    cudaMalloc(&out, 1 << 24);
    cudaMalloc(&cyc, 64 * 8);
    const int n = 4096;
    chain<1><<<1, 32>>>(out, n, cyc);
    cudaDeviceSynchronize();
    chain<1><<<1, 32>>>(out, n, cyc);
    cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("1 warp, dependent chain: %.1f cycles per hash\n", (double)h[0] / n);
    chain<4><<<1, 32>>>(out, n, cyc);
    cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("1 warp, 4 chains: %.1f cycles per hash\n", (double)h[0] / n / 4);
    chain<1><<<1, 1024>>>(out, n, cyc);
    cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("32 warps on one SM, 1 chain each: %.1f cycles per warp-hash (SM throughput %.2f warp-hashes/kcycle)\n",
           (double)h[0] / n, 32.0 * n / h[0] * 1000);
    return 0;
}

// DRAM fetch size and rate of random 4-byte loads by load flavour (the sampler's CSR `indices` reads):
// each thread makes `iters` independent random 4-byte loads from an 8 GB table. Run alone for the rate,
// under ncu (dram__bytes_read.sum) for the bytes fetched per load.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ldg tools/exp_ld_granularity.cu && /tmp/ldg
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint64_t x) {
    x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
    return (uint32_t)x;
}

template <int KIND>
__device__ __forceinline__ uint32_t ld(const uint32_t* p) {
    uint32_t v;
    if (KIND == 0) asm volatile("ld.global.nc.L2::64B.b32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (KIND == 1) asm volatile("ld.global.nc.b32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (KIND == 2) asm volatile("ld.global.cg.b32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (KIND == 3) asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (KIND == 4) asm volatile("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(v) : "l"(p));
    else asm volatile("ld.global.cs.b32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

template <int KIND, int U>
__global__ void rand_ld(const uint32_t* t, uint64_t words, int iters, uint32_t seed, uint32_t* sink) {
    const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t acc = 0;
    for (int it = 0; it < iters; it++) {
        uint32_t v[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint64_t r = ((uint64_t)hash32(tid * 1315423911ull + (uint64_t)(it * U + u) * 2654435761ull + seed) << 32 |
                                hash32(tid ^ ((uint64_t)(it * U + u) << 40) ^ seed)) % words;
            v[u] = ld<KIND>(t + r);
        }
#pragma unroll
        for (int u = 0; u < U; u++) acc += v[u];
    }
    if (acc == 0x12345678u) sink[0] = acc;
}

int main() {
    const uint64_t bytes = 8ull << 30, words = bytes / 4;
    uint32_t *t, *sink;
    cudaMalloc(&t, bytes);
    cudaMemset(t, 1, bytes);
    cudaMalloc(&sink, 4);
    const int blocks = 148 * 8, threads = 256, iters = 64;
    const double loads = (double)blocks * threads * iters * 8;
    const char* names[] = {"nc.L2::64B", "nc", "cg", "relaxed.gpu", "nc.L1::no_allocate", "cs"};
    for (int kind = 0; kind < 6; kind++) {
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        for (int rep = 0; rep < 2; rep++) {
            cudaEventRecord(a);
            switch (kind) {
                case 0: rand_ld<0, 8><<<blocks, threads>>>(t, words, iters, rep, sink); break;
                case 1: rand_ld<1, 8><<<blocks, threads>>>(t, words, iters, rep, sink); break;
                case 2: rand_ld<2, 8><<<blocks, threads>>>(t, words, iters, rep, sink); break;
                case 3: rand_ld<3, 8><<<blocks, threads>>>(t, words, iters, rep, sink); break;
                case 4: rand_ld<4, 8><<<blocks, threads>>>(t, words, iters, rep, sink); break;
                default: rand_ld<5, 8><<<blocks, threads>>>(t, words, iters, rep, sink); break;
            }
            cudaEventRecord(b);
            cudaEventSynchronize(b);
        }
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("%-20s %.2f G random 4-byte loads/s\n", names[kind], loads / (ms * 1e-3) / 1e9);
    }
    return 0;
}

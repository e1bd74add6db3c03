// Microbenchmark: throughput of the SSSP inner-loop access pattern on this GPU.
// Random 4-byte gathers (ld.global.cg) and random atomicMin into an array of
// `n` u32 (67 MB at n = 2^24, i.e. L2-sized like dist), with k independent
// accesses in flight per thread.  Prints G accesses/s per mode.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}

template <int K, int MODE>  // MODE 0 gather, 1 atomicMin, 2 gather + 10% atomicMin, 3 coalesced stream
__global__ void kern(uint32_t* a, uint32_t mask, uint64_t iters, uint32_t* sink) {
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t acc = 0, s = hash32(tid * 0x9E3779B9u + 17);
    for (uint64_t it = 0; it < iters; ++it) {
        uint32_t idx[K];
#pragma unroll
        for (int j = 0; j < K; ++j) { s = hash32(s + j); idx[j] = s & mask; }
        if (MODE == 3) {
#pragma unroll
            for (int j = 0; j < K; ++j) idx[j] = ((uint32_t)(it * K + j) * gridDim.x * blockDim.x + tid) & mask;
        }
        uint32_t v[K];
        if (MODE == 0 || MODE == 2 || MODE == 3) {
#pragma unroll
            for (int j = 0; j < K; ++j) v[j] = __ldcg(a + idx[j]);
#pragma unroll
            for (int j = 0; j < K; ++j) acc += v[j];
        }
        if (MODE == 1) {
#pragma unroll
            for (int j = 0; j < K; ++j) v[j] = atomicMin(a + idx[j], idx[j] ^ 0x5555u);
#pragma unroll
            for (int j = 0; j < K; ++j) acc += v[j];
        }
        if (MODE == 2) {
#pragma unroll
            for (int j = 0; j < K; ++j)
                if ((idx[j] & 15) == 0) acc += atomicMin(a + (idx[j] ^ 0x1234u) , acc);
        }
    }
    if (acc == 0x12345678u) sink[0] = acc;
}

template <int K, int MODE>
void run(const char* name, uint32_t* a, uint32_t mask, int grid, int block, uint32_t* sink) {
    const uint64_t iters = 64;
    kern<K, MODE><<<grid, block>>>(a, mask, 4, sink);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<K, MODE><<<grid, block>>>(a, mask, iters, sink);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
    const double acc = (double)grid * block * iters * K;
    printf("%-28s K=%d grid=%d block=%d : %8.1f G accesses/s (%.3f ms)\n", name, K, grid, block, acc / ms / 1e6, ms);
}

int main() {
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const uint32_t n = 1u << 24;
    uint32_t *a, *sink;
    cudaMalloc(&a, (size_t)n * 4); cudaMalloc(&sink, 64);
    cudaMemset(a, 0x7f, (size_t)n * 4);
    for (int bpsm : {2, 4, 8}) {
        const int grid = sms * bpsm, block = 256;
        run<4, 0>("gather L2-resident", a, n - 1, grid, block, sink);
        run<4, 1>("atomicMin random", a, n - 1, grid, block, sink);
        run<4, 2>("gather + 1/16 atomicMin", a, n - 1, grid, block, sink);
        run<4, 3>("coalesced (reference)", a, n - 1, grid, block, sink);
    }
    run<8, 0>("gather L2-resident", a, n - 1, sms * 8, 256, sink);
    run<16, 0>("gather L2-resident", a, n - 1, sms * 8, 256, sink);
    // 4 GB array: gathers that miss L2
    uint32_t* big; const uint32_t nb = 1u << 30;
    if (cudaMalloc(&big, (size_t)nb * 4) == cudaSuccess) {
        run<4, 0>("gather 4 GB (HBM)", big, nb - 1, sms * 8, 256, sink);
        run<8, 0>("gather 4 GB (HBM)", big, nb - 1, sms * 8, 256, sink);
    }
    printf("SMs=%d\n", sms);
    return 0;
}

// Microbenchmark: throughput of atomics on a FEW hot addresses (the bucket ring's
// per-bucket counters) on this GPU.  One lane per warp issues the atomic (as the
// ADDS kernels do: one counter update per warp/CTA batch).  Modes:
//   0  returning atomicAdd (u64) on H addresses (claim / reserve)
//   1  non-returning RED add (u64) on H addresses (publish / done)
//   2  relaxed load of H addresses (idle polling of avail/head lines)
// Prints G ops/s for H = 1, 2, 8, 32 counters (each on its own 128-B line).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE>
__global__ void kern(unsigned long long* c, int H, int iters, unsigned long long* sink) {
    const int lane = threadIdx.x & 31;
    if (lane != 0) return;
    const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    unsigned long long acc = 0;
    for (int i = 0; i < iters; ++i) {
        unsigned long long* p = c + (size_t)((w + i) % H) * 16;
        if (MODE == 0) acc += atomicAdd(p, 1ull);
        if (MODE == 1) atomicAdd(p, 1ull), acc += i;
        if (MODE == 2) {
            unsigned long long v;
            asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
            acc += v;
        }
    }
    if (acc == 0x123456789ull) sink[0] = acc;
}

template <int MODE>
void run(const char* name, unsigned long long* c, unsigned long long* sink, int H, int grid, int block) {
    const int iters = 256;
    kern<MODE><<<grid, block>>>(c, H, 4, sink);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    kern<MODE><<<grid, block>>>(c, H, iters, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    const double ops = (double)grid * (block / 32) * iters;
    printf("%-22s H=%2d warps=%6d  %8.3f G ops/s  (%.1f M ops/s per counter)\n", name, H, grid * (block / 32),
           ops / ms / 1e6, ops / ms / 1e3 / H);
}

int main() {
    unsigned long long *c, *sink;
    cudaMalloc(&c, 64 * 128);
    cudaMalloc(&sink, 8);
    cudaMemset(c, 0, 64 * 128);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int H : {1, 2, 8, 32}) {
        run<0>("returning atomicAdd", c, sink, H, sms * 2, 512);
        run<1>("RED add", c, sink, H, sms * 2, 512);
        run<2>("relaxed load", c, sink, H, sms * 2, 512);
    }
    // fewer issuers (CTA-granular: one issuing warp per CTA)
    for (int H : {1, 8}) {
        run<0>("returning (1 warp/CTA)", c, sink, H, sms * 2, 32);
        run<1>("RED (1 warp/CTA)", c, sink, H, sms * 2, 32);
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("status: %s\n", cudaGetErrorString(e));
    return 0;
}

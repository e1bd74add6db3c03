// Does an L2 policy protect a 67 MB randomly-gathered array (like dist) from a
// competing coalesced 4 GB stream (like the arcs)?  Each thread alternates K
// random gathers on A with K coalesced stream loads on B.  Variants: stream
// hint (normal / evict_first / no_allocate-L1), gather hint (normal / evict_last),
// persisting set-aside on/off.  Reports gathers/s and the kernel time.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}
__device__ __forceinline__ unsigned long long pol_first() { unsigned long long p; asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ unsigned long long pol_last(float f) { unsigned long long p; asm volatile("createpolicy.fractional.L2::evict_last.L2::evict_unchanged.b64 %0, %1;" : "=l"(p) : "f"(f)); return p; }

template <int SH, int GH>  // SH: 0 normal, 1 evict_first;  GH: 0 normal .cg, 1 evict_last
__global__ void kern(const uint32_t* a, uint32_t amask, const uint2* b, unsigned long long bn, uint64_t iters,
                     uint32_t* sink, float frac) {
    const unsigned long long T = (unsigned long long)gridDim.x * blockDim.x;
    const unsigned long long tid = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
    const unsigned long long pf = pol_first(), pl = pol_last(frac);
    uint32_t acc = 0, s = hash32((uint32_t)tid * 0x9E3779B9u + 17);
    unsigned long long bi = tid;
    for (uint64_t it = 0; it < iters; ++it) {
        uint32_t v[4];
        uint2 w[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            s = hash32(s + j);
            const uint32_t* ap = a + (s & amask);
            if (GH) asm volatile("ld.global.cg.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v[j]) : "l"(ap), "l"(pl));
            else v[j] = __ldcg(ap);
            const uint2* bp = b + (bi % bn);
            bi += T;
            if (SH) asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0,%1}, [%2], %3;" : "=r"(w[j].x), "=r"(w[j].y) : "l"(bp), "l"(pf));
            else w[j] = __ldg(bp);
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) acc += v[j] + w[j].x;
    }
    if (acc == 0x12345678u) sink[0] = acc;
}

template <int SH, int GH>
void run(const char* name, const uint32_t* a, uint32_t amask, const uint2* b, unsigned long long bn, uint32_t* sink,
         int sms, float frac) {
    const int grid = sms * 8, block = 256;
    const uint64_t iters = 128;
    kern<SH, GH><<<grid, block>>>(a, amask, b, bn, 8, sink, frac);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<SH, GH><<<grid, block>>>(a, amask, b, bn, iters, sink, frac);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
    const double g = (double)grid * block * iters * 4;
    printf("%-44s %8.1f G gathers/s  (+ same count of stream loads, %.2f GB streamed)  %.3f ms\n", name, g / ms / 1e6,
           g * 8 / 1e9, ms);
}

int main() {
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceProp prop; cudaGetDeviceProperties(&prop, 0);
    const uint32_t n = 1u << 24;             // 64 MiB of u32 (67 MB)
    const unsigned long long bn = 1ull << 29;  // 4 GiB of uint2
    uint32_t *a, *sink; uint2* b;
    cudaMalloc(&a, (size_t)n * 4); cudaMalloc(&sink, 64); cudaMalloc(&b, bn * 8);
    cudaMemset(a, 1, (size_t)n * 4); cudaMemset(b, 2, bn * 8);
    for (int persist = 0; persist < 2; ++persist) {
        size_t lim = persist ? (size_t)prop.persistingL2CacheMaxSize : 0;
        cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, lim);
        size_t got = 0; cudaDeviceGetLimit(&got, cudaLimitPersistingL2CacheSize);
        printf("--- persisting set-aside = %zu bytes\n", got);
        run<0, 0>("stream normal,      gather normal", a, n - 1, b, bn, sink, sms, 1.0f);
        run<1, 0>("stream evict_first, gather normal", a, n - 1, b, bn, sink, sms, 1.0f);
        run<0, 1>("stream normal,      gather evict_last", a, n - 1, b, bn, sink, sms, 1.0f);
        run<1, 1>("stream evict_first, gather evict_last", a, n - 1, b, bn, sink, sms, 1.0f);
        run<1, 1>("stream evict_first, gather evict_last f=.8", a, n - 1, b, bn, sink, sms, 0.8f);
    }
    // gathers alone, for reference
    run<0, 0>("(no stream) -- see gather_bench", a, n - 1, b, 1, sink, sms, 1.0f);
    return 0;
}

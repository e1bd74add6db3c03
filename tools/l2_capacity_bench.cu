// How much of the 126 MB L2 can a randomly gathered array use on B200?
// Random 4-byte gathers (ld.global.cg, K in flight per thread, all SMs) over an
// array of S MB, S swept from 8 to 160 MB.  If the two dies' L2s each keep their
// own copy of lines their SMs read, the hit rate falls once S passes one die's
// share (~63 MB), not the full 126 MB.  Run plain for G/s and under
//   ncu --metrics lts__t_sector_hit_rate.pct,dram__bytes_read.sum
// for the hit rate per size.  Mode 1 = atomicMin instead of loads (atomics are
// resolved at the line's home slice), mode 2 = loads from SMs with even %smid
// only touching the lower half and odd the upper half (a die split, if the SM
// numbering alternates dies), mode 3 = lower half for smid < SMs/2.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}
__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }

template <int MODE>
__global__ void kern(uint32_t* a, uint32_t n, uint64_t iters, uint32_t* sink, unsigned nsm) {
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t acc = 0, s = hash32(tid * 0x9E3779B9u + 17);
    const unsigned sm = smid();
    uint32_t lo = 0, span = n;
    if (MODE == 2) { span = n / 2; lo = (sm & 1) ? span : 0; }
    if (MODE == 3) { span = n / 2; lo = (sm >= nsm / 2) ? span : 0; }
    for (uint64_t it = 0; it < iters; ++it) {
        uint32_t idx[8], v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) { s = hash32(s + j); idx[j] = lo + (uint32_t)(((unsigned long long)s * span) >> 32); }
        if (MODE == 1) {
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = atomicMin(a + idx[j], 0x7f000000u);
        } else {
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = __ldcg(a + idx[j]);
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) acc += v[j];
    }
    if (acc == 0x12345678u) sink[0] = acc;
}

template <int MODE>
double run(uint32_t* a, uint32_t n, uint32_t* sink, int sms) {
    const int grid = sms * 8, block = 256;
    const uint64_t iters = 48;
    kern<MODE><<<grid, block>>>(a, n, 16, sink, sms);  // warm the cache
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<MODE><<<grid, block>>>(a, n, iters, sink, sms);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
    return (double)grid * block * iters * 8 / ms / 1e6;
}

int main() {
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceProp prop; cudaGetDeviceProperties(&prop, 0);
    printf("SMs=%d l2=%d B persistingMax=%d B\n", sms, prop.l2CacheSize, prop.persistingL2CacheMaxSize);
    uint32_t *a, *sink;
    const size_t maxb = 160ull << 20;
    cudaMalloc(&a, maxb); cudaMalloc(&sink, 64);
    cudaMemset(a, 0x7f, maxb);
    for (int mb : {8, 16, 32, 48, 56, 64, 72, 80, 96, 112, 128, 160}) {
        const uint32_t n = (uint32_t)(((size_t)mb << 20) / 4);
        const double g0 = run<0>(a, n, sink, sms);
        const double g1 = run<1>(a, n, sink, sms);
        const double g2 = run<2>(a, n, sink, sms);
        const double g3 = run<3>(a, n, sink, sms);
        printf("S=%4d MB  gather %7.1f  atomicMin %7.1f  split-even/odd %7.1f  split-lo/hi %7.1f  G/s\n", mb, g0, g1,
               g2, g3);
    }
    return 0;
}

// Device facts relevant to L2 residency (persisting set-aside) -- run on the GPU box.
#include <cstdio>
#include <cuda_runtime.h>
int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    printf("name=%s sms=%d l2=%d persistingL2CacheMaxSize=%d accessPolicyMaxWindowSize=%d smemPerSM=%zu smemPerBlockOptin=%zu regsPerSM=%d clock=%d memclk=%d buswidth=%d\n",
           p.name, p.multiProcessorCount, p.l2CacheSize, p.persistingL2CacheMaxSize, p.accessPolicyMaxWindowSize,
           p.sharedMemPerMultiprocessor, p.sharedMemPerBlockOptin, p.regsPerMultiprocessor, p.clockRate, p.memoryClockRate, p.memoryBusWidth);
    size_t v = 0;
    cudaDeviceGetLimit(&v, cudaLimitPersistingL2CacheSize);
    printf("current persisting limit=%zu\n", v);
    cudaError_t e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, p.persistingL2CacheMaxSize);
    cudaDeviceGetLimit(&v, cudaLimitPersistingL2CacheSize);
    printf("set -> %s, now %zu\n", cudaGetErrorString(e), v);
    return 0;
}

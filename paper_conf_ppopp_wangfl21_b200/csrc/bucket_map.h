// bucket_map.h -- the bucket ring's priority mapping, shared by the persistent
// kernel and the host-callable sssp_bucket_offset() (unit-tested on CPU).
//
// PAPER.md P:174 (§5.4): "Our work queue consists of a fixed number of 32
// buckets, managed as a circular priority queue"; P:83 (§3.2): vertices whose
// priorities "differ by up to a constant called Delta" share a bucket
// (§5.5): "vertices out of range will be clipped to the last bucket".
// Reading (R4/R5): Delta = 2^k, an item of distance d belongs to
// absolute bucket floor(d / Delta) = d >> k; the ring's head holds absolute
// bucket `head`; items below the head go to the head, items at or beyond
// head + B - 1 are clipped into the tail.
#pragma once
#include <stdint.h>

#if defined(__CUDACC__)
#define ADDS_HD __host__ __device__ __forceinline__
#else
#define ADDS_HD static inline
#endif

ADDS_HD uint32_t adds_bucket_offset(uint64_t d, uint32_t k, uint64_t head, uint32_t nb) {
    uint64_t j = k >= 64 ? 0 : (d >> k);
    if (j <= head) return 0u;
    uint64_t off = j - head;
    return off >= (uint64_t)(nb - 1) ? nb - 1 : (uint32_t)off;
}

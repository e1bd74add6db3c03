// certify_kernels.cuh -- O(n + m) GPU certificate of a distance vector (sssp_certify).
//
// SURVEY.md §8(c) "What pins each part": a vector d is the exact shortest-distance
// vector from s iff
//   (i)   d[s] = 0;
//   (ii)  no arc is violated: for every arc (u, v, w) with d[u] finite,
//         d[v] <= d[u] (+) w  (so d is never above the true distances);
//   (iii) every finite v is reachable from s through TIGHT arcs, d[u] (+) w == d[v]
//         (so d is the length of some path: never below the true distances);
//   (iv)  unreachable <=> UINT64_MAX (float graphs: +inf).
// (+) is the integer sum, or the round-to-nearest binary32 sum for float32-weight
// graphs (NEXT-3; fl(a + w) is monotone in a, so the same argument holds).
//
// (iii) is checked without a BFS in the common case: a vertex with a tight in-arc
// from a vertex of strictly smaller distance is "anchored" by that arc; by induction
// on the distance every finite vertex is then reachable through tight arcs, as long
// as every finite vertex is anchored.  Tight arcs between EQUAL distances (zero
// weights, or float absorption) are resolved by iterating "a tight equal-distance
// arc from an anchored vertex anchors its head" to a fixed point (launched only when
// such arcs exist; none do on the BASELINE configs, whose weights are >= 1).
//
// This is the checker of the GPU result used by the tests on every source of the
// multi-source batch (config 5); it shares nothing with the SSSP kernels but the CSR
// layout.  The rows are scattered into the library's internal vertex order first
// (locality relabeling, D15).
#pragma once
#include <cstdint>

namespace adds {

struct CertState {
    unsigned long long violated;      // arcs breaking (ii)
    unsigned long long first_violated;// smallest internal tail vertex of a violated arc (~0 = none)
    unsigned long long unanchored;    // finite vertices not reachable through tight arcs (iii)
    unsigned long long first_unanchored;
    unsigned long long reach_v, reach_e;  // V_dij, E_dij of the vector
    unsigned long long equal_tight;   // tight arcs between equal distances (fixpoint needed)
    unsigned long long changed;       // fixpoint iteration flag
    unsigned long long bad_inf;       // (iv): an 'unreachable' entry that is not the exact marker
    unsigned long long source_bad;    // (i)
};

template <bool kF>
__device__ __forceinline__ unsigned long long cert_inf() {
    return kF ? 0x7F800000ull : ~0ull;
}
// d (+) w, saturating at the infinity marker (a corrupt near-2^64 entry cannot wrap)
template <bool kF>
__device__ __forceinline__ unsigned long long cert_sum(unsigned long long d, unsigned w) {
    if constexpr (kF) {
        const float s = __fadd_rn(__uint_as_float((unsigned)d), __uint_as_float(w));
        const unsigned b = __float_as_uint(s);
        return b >= 0x7F800000u ? 0x7F800000ull : (unsigned long long)b;
    } else {
        const unsigned long long s = d + (unsigned long long)w;
        return s < d ? ~0ull : s;
    }
}

// dint[perm[v]] = caller_dist[v] (perm nullable = identity); anchors[] cleared; (i), (iv)
template <bool kF>
__global__ void certify_scatter_kernel(const void* __restrict__ caller_dist, unsigned long long* __restrict__ dint,
                                       const unsigned* __restrict__ perm, unsigned n, unsigned source,
                                       unsigned* __restrict__ anchors, CertState* st) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    const unsigned long long t0 = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
    for (unsigned long long v = t0; v < n; v += stride) {
        unsigned long long d;
        if constexpr (kF) {
            const unsigned b = ((const unsigned*)caller_dist)[v];
            // +inf is the unreachable marker; NaN or negative values are never distances
            if (b > 0x7F800000u) atomicAdd(&st->bad_inf, 1ull);
            d = b >= 0x7F800000u ? 0x7F800000ull : (unsigned long long)b;
        } else {
            d = ((const unsigned long long*)caller_dist)[v];
        }
        const unsigned long long iv = perm ? perm[v] : v;
        dint[iv] = d;
        if (v == source && d != 0) atomicAdd(&st->source_bad, 1ull);
    }
    const unsigned long long nw = ((unsigned long long)n + 31) / 32;
    for (unsigned long long i = t0; i < nw; i += stride) anchors[i] = 0u;
}

// (ii) + anchors by strictly-smaller tight in-arcs; one warp per row, lanes over its arcs
template <bool kF>
__global__ void certify_arcs_kernel(const unsigned long long* __restrict__ dint, const unsigned long long* __restrict__ off,
                                    const uint2* __restrict__ adj, unsigned n, unsigned src_int,
                                    unsigned* __restrict__ anchors, CertState* st) {
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long nw = (unsigned long long)gridDim.x * blockDim.x / 32;
    const unsigned long long inf = cert_inf<kF>();
    unsigned long long viol = 0, eq = 0, first = ~0ull;
    for (unsigned long long u = ((unsigned long long)blockIdx.x * blockDim.x + threadIdx.x) / 32; u < n; u += nw) {
        if (u == src_int && lane == 0) atomicOr(&anchors[u >> 5], 1u << (u & 31));
        const unsigned long long du = dint[u];
        if (du >= inf) continue;  // (ii) constrains arcs out of finite vertices only
        const unsigned long long b = off[u], e = off[u + 1];
        for (unsigned long long k = b + lane; k < e; k += 32) {
            const uint2 a = adj[k];
            const unsigned long long nd = cert_sum<kF>(du, a.y);
            const unsigned long long dv = dint[a.x];
            if (dv > nd) {
                ++viol;
                first = u < first ? u : first;
            } else if (dv == nd && nd < inf) {
                if (du < dv) atomicOr(&anchors[a.x >> 5], 1u << (a.x & 31));
                else ++eq;
            }
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        viol += __shfl_xor_sync(0xffffffffu, viol, o);
        eq += __shfl_xor_sync(0xffffffffu, eq, o);
        first = min(first, __shfl_xor_sync(0xffffffffu, first, o));
    }
    if (lane == 0) {
        if (viol) {
            atomicAdd(&st->violated, viol);
            atomicMin(&st->first_violated, first);
        }
        if (eq) atomicAdd(&st->equal_tight, eq);
    }
}

// one fixpoint round over tight equal-distance arcs: an anchored tail anchors its head
template <bool kF>
__global__ void certify_equal_kernel(const unsigned long long* __restrict__ dint, const unsigned long long* __restrict__ off,
                                     const uint2* __restrict__ adj, unsigned n, unsigned* __restrict__ anchors,
                                     CertState* st) {
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long nw = (unsigned long long)gridDim.x * blockDim.x / 32;
    const unsigned long long inf = cert_inf<kF>();
    unsigned changed = 0;
    for (unsigned long long u = ((unsigned long long)blockIdx.x * blockDim.x + threadIdx.x) / 32; u < n; u += nw) {
        const unsigned long long du = dint[u];
        if (du >= inf || !((__ldcg(&anchors[u >> 5]) >> (u & 31)) & 1u)) continue;
        const unsigned long long b = off[u], e = off[u + 1];
        for (unsigned long long k = b + lane; k < e; k += 32) {
            const uint2 a = adj[k];
            if (dint[a.x] == du && cert_sum<kF>(du, a.y) == du) {
                const unsigned bit = 1u << (a.x & 31);
                if (!(__ldcg(&anchors[a.x >> 5]) & bit) && !(atomicOr(&anchors[a.x >> 5], bit) & bit)) changed = 1;
            }
        }
    }
    if (__any_sync(0xffffffffu, changed) && lane == 0) atomicAdd(&st->changed, 1ull);
}

// (iii): every finite vertex anchored; V_dij / E_dij of the vector
template <bool kF>
__global__ void certify_check_kernel(const unsigned long long* __restrict__ dint, const unsigned long long* __restrict__ off,
                                     unsigned n, const unsigned* __restrict__ anchors, CertState* st) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    const unsigned long long inf = cert_inf<kF>();
    unsigned long long un = 0, rv = 0, re = 0, first = ~0ull;
    for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        if (dint[v] >= inf) continue;
        ++rv;
        re += off[v + 1] - off[v];
        if (!((anchors[v >> 5] >> (v & 31)) & 1u)) {
            ++un;
            first = v < first ? v : first;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        un += __shfl_xor_sync(0xffffffffu, un, o);
        rv += __shfl_xor_sync(0xffffffffu, rv, o);
        re += __shfl_xor_sync(0xffffffffu, re, o);
        first = min(first, __shfl_xor_sync(0xffffffffu, first, o));
    }
    if ((threadIdx.x & 31) == 0) {
        if (un) {
            atomicAdd(&st->unanchored, un);
            atomicMin(&st->first_unanchored, first);
        }
        if (rv) {
            atomicAdd(&st->reach_v, rv);
            atomicAdd(&st->reach_e, re);
        }
    }
}

}  // namespace adds

// aux_kernels.cuh -- create-time and per-run helper kernels (grid-stride, sm_100a).
//   validate_csr   O(n+m) CSR checks (§8(b) "Validation at create")
//   interleave     {col, w} -> 8-byte arcs + sum/max of weights (initial Delta)
//   init_run       dist = inf, dist[s] = 0, ring counters reset, source item pushed (§8(a) A3)
//   finalize       widen dist to uint64 (inf -> UINT64_MAX) + reach / E_dij / max (§8(a) A10)
#pragma once
#include "common.cuh"

namespace adds {

__global__ void validate_csr_kernel(const unsigned long long* __restrict__ off, const unsigned* __restrict__ col,
                                    unsigned n, unsigned long long m, unsigned long long* bad) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        if (off[v] > off[v + 1]) atomicMin(&bad[0], v);
    for (unsigned long long e = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; e < m; e += stride)
        if (col[e] >= n) atomicMin(&bad[1], e);
}

// A run's status block to mapped pinned host memory: posted PCIe writes, not a copy-engine job, so
// the host's wait for a finished run never queues behind a large device->host copy in flight
// (the host-output batch overlaps those with the next sources, sssp_lib.cu run_concurrent).
__global__ void status_copy_kernel(const unsigned long long* __restrict__ src, unsigned long long* dst, unsigned words) {
    for (unsigned i = threadIdx.x; i < words; i += blockDim.x) ((volatile unsigned long long*)dst)[i] = __ldcg(src + i);
    __threadfence_system();
}

// Per-vertex row records {row begin, degree} in 32 bits for graphs with m < 2^32: the
// throughput kernel's pop reads one aligned 8-byte record instead of two 8-byte offsets.
__global__ void rows32_kernel(const unsigned long long* __restrict__ off, unsigned n, uint2* __restrict__ rows) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        rows[v] = make_uint2((unsigned)off[v], (unsigned)(off[v + 1] - off[v]));
}

__global__ void interleave_kernel(const unsigned* __restrict__ col, const unsigned* __restrict__ w,
                                  uint2* __restrict__ adj, unsigned long long m, unsigned long long* sum_w,
                                  unsigned* max_w) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned long long s = 0;
    unsigned mx = 0;
    for (unsigned long long e = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; e < m; e += stride) {
        const unsigned ww = w[e];
        adj[e] = make_uint2(col[e], ww);
        s += ww;
        mx = ww > mx ? ww : mx;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        s += __shfl_xor_sync(0xffffffffu, s, o);
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(sum_w, s);
        atomicMax(max_w, mx);
    }
}

// Chunked bucket storage (nullable): chunk tables (nb x tab_stride entries), per-chunk read
// counts and the free ring are reset; the source's chunk is chunk 0.
struct ChunkInit {
    unsigned* ctab = nullptr;
    unsigned tab_stride = 0, nb = 0;
    unsigned* chunk_used = nullptr;
    unsigned* free_ring = nullptr;
    unsigned pool_chunks = 0;
    ChunkPool* pool = nullptr;
};
template <typename DistT>
__global__ void init_run_kernel(DistT* __restrict__ dist, unsigned n, unsigned source, Ctl* ctl, BucketCtl* bk,
                                char* ring, unsigned long long cap, Head h0, unsigned* expanded,
                                unsigned short* filt, ChunkInit ci) {
    using IT = ItemT<DistT>;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        dist[v] = (v == source) ? (DistT)0 : DistInf<DistT>::value;
    if (filt)
        for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
            filt[v] = (v == source) ? (unsigned short)0 : (unsigned short)0xFFFFu;
    const unsigned long long nw = ((unsigned long long)n + 31) / 32;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += stride)
        expanded[i] = 0u;
    if (ci.ctab) {
        const unsigned long long nt = (unsigned long long)ci.nb * ci.tab_stride;
        const unsigned hs = meta_hs(h0.meta);
        for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < nt; i += stride)
            ci.ctab[i] = (i == (unsigned long long)hs * ci.tab_stride) ? 1u : 0u;  // chunk 0: the source's
        for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < ci.pool_chunks;
             i += stride) {
            ci.chunk_used[i] = 0u;
            ci.free_ring[i] = 0u;
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            ci.pool->fresh.v = 1;
            ci.pool->freserve.v = ci.pool->favail.v = ci.pool->fclaim.v = 0;
        }
    }
    if (blockIdx.x == 0) {
        const unsigned t = threadIdx.x;
        if (t == kSplitQ) bk[t].reserve.v = bk[t].avail.v = bk[t].claim.v = bk[t].done.v = bk[t].local.v = 0;
        if (t < kMaxBuckets) {
            bk[t].reserve.v = 0;
            bk[t].avail.v = 0;
            bk[t].claim.v = 0;
            bk[t].done.v = 0;
            bk[t].local.v = 0;
            if (t == meta_hs(h0.meta)) {  // the source item: bucket 0 = head ("initially ... infinity")
                // (chunked storage: item 0 of the head slot is item 0 of chunk 0)
                IT::store(ring + (ci.ctab ? (size_t)0 : (size_t)t * cap * IT::kBytes), IT::make(source, 0ull));
                bk[t].reserve.v = 1;
                bk[t].avail.v = 1;
            }
        }
        if (t == 0) {
            ctl->head = h0;
            ctl->status = 0;
            ctl->trace_count = 0;
            ctl->head_switches = 0;
            ctl->delta_changes = 0;
            ctl->t_start = globaltimer();
            ctl->g_exp = ctl->g_first = ctl->exp_mark = ctl->first_mark = 0;
            ctl->g_push = ctl->g_clip = ctl->push_mark = ctl->clip_mark = 0;
            ctl->g_busy = 0;
            ctl->last_waste = 0;
            ctl->last_ctl_ns = ctl->t_start;
            ctl->st_vertices = ctl->st_edges = ctl->st_pushes = ctl->st_stale = ctl->st_local = 0;
            ctl->reach_v = ctl->reach_e = ctl->max_dist = 0;
            for (int i = 0; i < (int)kProfCounters; ++i) ctl->prof[i] = 0;
        }
    }
}

// perm (nullable): internal id of each caller vertex id (locality relabeling, D15);
// the output is written in caller order, coalesced, gathering from the internal array
template <typename DistT>
__global__ void finalize_kernel(const DistT* __restrict__ dist, unsigned long long* __restrict__ out, unsigned n,
                                const unsigned long long* __restrict__ off, Ctl* ctl,
                                const unsigned* __restrict__ perm = nullptr) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned long long rv = 0, re = 0, mx = 0;
    for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        const unsigned long long iv = perm ? perm[v] : v;
        const DistT d = dist[iv];
        if (d == DistInf<DistT>::value) {
            out[v] = ~0ull;
        } else {
            out[v] = (unsigned long long)d;
            rv += 1;
            re += off[iv + 1] - off[iv];
            mx = (unsigned long long)d > mx ? (unsigned long long)d : mx;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        rv += __shfl_xor_sync(0xffffffffu, rv, o);
        re += __shfl_xor_sync(0xffffffffu, re, o);
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    if ((threadIdx.x & 31) == 0 && rv) {
        atomicAdd(&ctl->reach_v, rv);
        atomicAdd(&ctl->reach_e, re);
        atomicMax(&ctl->max_dist, mx);
    }
}

// float32-weight graphs (NEXT-3): validate (no negative or NaN weight), fold
// -0.0 into +0.0 (bit order must equal value order), interleave, max weight
__global__ void interleave_f32_kernel(const unsigned* __restrict__ col, unsigned* __restrict__ wbits,
                                      uint2* __restrict__ adj, unsigned long long m, unsigned long long* bad_w,
                                      unsigned* max_w) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned mx = 0;
    for (unsigned long long e = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; e < m; e += stride) {
        unsigned wb = wbits[e];
        if (wb == 0x80000000u) wb = 0u;                       // -0.0 -> +0.0
        if ((wb & 0x80000000u) || (wb & 0x7FFFFFFFu) > 0x7F800000u) atomicMin(bad_w, e);  // negative / NaN
        adj[e] = make_uint2(col[e], wb);
        if (wb <= 0x7F800000u) mx = wb > mx ? wb : mx;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if ((threadIdx.x & 31) == 0) atomicMax(max_w, mx);
}

__global__ void finalize_f32_kernel(const unsigned* __restrict__ dist, float* __restrict__ out, unsigned n,
                                    const unsigned long long* __restrict__ off, Ctl* ctl,
                                    const unsigned* __restrict__ perm = nullptr) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned long long rv = 0, re = 0, mx = 0;
    for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        const unsigned long long iv = perm ? perm[v] : v;
        const unsigned d = dist[iv];
        if (d >= 0x7F800000u) {  // never reached (internal sentinel) or +inf
            out[v] = __uint_as_float(0x7F800000u);
        } else {
            out[v] = __uint_as_float(d);
            rv += 1;
            re += off[iv + 1] - off[iv];
            mx = d > mx ? d : mx;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        rv += __shfl_xor_sync(0xffffffffu, rv, o);
        re += __shfl_xor_sync(0xffffffffu, re, o);
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    if ((threadIdx.x & 31) == 0 && rv) {
        atomicAdd(&ctl->reach_v, rv);
        atomicAdd(&ctl->reach_e, re);
        atomicMax(&ctl->max_dist, mx);
    }
}

// ---------------------------------------------------------------- locality relabeling (D15)
// in-degree of every vertex (the number of arcs that gather/atomically update its dist)
__global__ void indegree_kernel(const uint2* __restrict__ adj, unsigned long long m, unsigned* __restrict__ indeg) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long e = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; e < m; e += stride)
        atomicAdd(&indeg[adj[e].x], 1u);
}
// sort keys: descending in-degree (ascending ~indeg), ties by id (stable sort of an iota)
__global__ void relabel_keys_kernel(const unsigned* __restrict__ indeg, unsigned n, unsigned* __restrict__ key,
                                    unsigned* __restrict__ iota) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        key[v] = ~indeg[v];
        iota[v] = (unsigned)v;
    }
}
// new_of_old[old_of_new[i]] = i; degree of internal vertex i
__global__ void relabel_inverse_kernel(const unsigned* __restrict__ old_of_new, unsigned n,
                                       const unsigned long long* __restrict__ off, unsigned* __restrict__ new_of_old,
                                       unsigned long long* __restrict__ deg_new) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const unsigned o = old_of_new[i];
        new_of_old[o] = (unsigned)i;
        deg_new[i] = off[o + 1] - off[o];
    }
}
// one warp per internal row: copy the old row's arcs, renaming their heads
__global__ void relabel_arcs_kernel(const unsigned* __restrict__ old_of_new, const unsigned* __restrict__ new_of_old,
                                    unsigned n, const unsigned long long* __restrict__ off,
                                    const unsigned long long* __restrict__ off_new, const uint2* __restrict__ adj,
                                    uint2* __restrict__ adj_new) {
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long nw = (unsigned long long)gridDim.x * blockDim.x / 32;
    for (unsigned long long i = ((unsigned long long)blockIdx.x * blockDim.x + threadIdx.x) / 32; i < n; i += nw) {
        const unsigned o = old_of_new[i];
        const unsigned long long b = off[o], e = off[o + 1], nb = off_new[i];
        for (unsigned long long k = b + lane; k < e; k += 32) {
            const uint2 a = adj[k];
            adj_new[nb + (k - b)] = make_uint2(new_of_old[a.x], a.y);
        }
    }
}

}  // namespace adds

// nearfar_kernel.cuh -- BSP Near-Far ablation (the paper's
// comparison system NF), selectable with
// options.algorithm = SSSP_ALGO_NEAR_FAR.
//
// Two piles, double-buffered, bulk-synchronous ("it uses just two
// buckets, known as Near and Far ... supersteps separated by barrier
// synchronization ... each bucket [is] double buffered"):
//   superstep: every item of Near[cur] is expanded in parallel; an improved
//     vertex goes to Near[nxt] if its distance is below the split, else to Far;
//     grid barrier; swap.
//   when Near is empty: split += Delta and the Far pile is partitioned (stale
//     items dropped): items below the split -> Near, the rest -> the other Far
//     buffer; grid barrier.
//   done when both piles are empty.
// One cooperative persistent launch; the barrier is cg::grid_group::sync().
// Items are {vertex, distance-at-push} like the ADDS ring.  Expansion is
// warp-centric: rows with >= 32 arcs are processed by the whole warp (coalesced),
// shorter rows by their own lane.
#pragma once
#include <cooperative_groups.h>

#include "common.cuh"

namespace adds {

struct NFCounters {
    Counter near_cnt[2];
    Counter far_cnt[2];
    Counter supersteps;
};

template <typename DistT>
struct NFParams {
    const unsigned long long* __restrict__ off;
    const uint2* __restrict__ adj;
    DistT* dist;
    unsigned long long* near[2];  // items: v | d << 32 (u32 dist) or 16-byte pairs (u64)
    unsigned long long* far[2];
    NFCounters* cnt;
    Ctl* ctl;
    unsigned long long cap;  // items per pile buffer
    unsigned long long delta;
    unsigned long long timeout_ns;
};

template <typename DistT>
struct NFItem;
template <>
struct NFItem<uint32_t> {
    static constexpr int kWords = 1;
    __device__ static void put(unsigned long long* base, unsigned long long i, unsigned v, unsigned long long d) {
        base[i] = (unsigned long long)v | (d << 32);
    }
    __device__ static void get(const unsigned long long* base, unsigned long long i, unsigned& v, unsigned long long& d) {
        const unsigned long long x = base[i];
        v = (unsigned)x;
        d = x >> 32;
    }
};
template <>
struct NFItem<unsigned long long> {
    static constexpr int kWords = 2;
    __device__ static void put(unsigned long long* base, unsigned long long i, unsigned v, unsigned long long d) {
        base[2 * i] = v;
        base[2 * i + 1] = d;
    }
    __device__ static void get(const unsigned long long* base, unsigned long long i, unsigned& v, unsigned long long& d) {
        v = (unsigned)base[2 * i];
        d = base[2 * i + 1];
    }
};

// warp-aggregated append of one item per active lane to pile `pile` (counter c)
template <typename DistT>
__device__ __forceinline__ void nf_append(const NFParams<DistT>& p, unsigned long long* pile, Counter* c, bool want,
                                          unsigned v, unsigned long long d) {
    const unsigned m = __ballot_sync(0xffffffffu, want);
    if (!m) return;
    const int lane = threadIdx.x & 31, leader = __ffs(m) - 1;
    unsigned long long base = 0;
    if (lane == leader) base = atomicAdd(&c->v, (unsigned long long)__popc(m));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (want) {
        unsigned lt;
        asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
        const unsigned long long i = base + __popc(m & lt);
        if (i < p.cap) NFItem<DistT>::put(pile, i, v, d);
        else atomicOr(&p.ctl->status, kStRingOverflow);
    }
}

template <typename DistT>
__global__ void __launch_bounds__(256) near_far_kernel(const NFParams<DistT> p) {
    namespace cg = cooperative_groups;
    cg::grid_group grid = cg::this_grid();
    constexpr unsigned long long kInf = (unsigned long long)DistInf<DistT>::value;
    const int lane = threadIdx.x & 31;
    const unsigned long long gwarp = ((unsigned long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const unsigned long long nwarps = ((unsigned long long)gridDim.x * blockDim.x) >> 5;
    const unsigned long long gtid = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
    const unsigned long long nthreads = (unsigned long long)gridDim.x * blockDim.x;
    unsigned long long split = p.delta;
    int cur = 0, fcur = 0;
    unsigned long long c_vert = 0, c_edges = 0, c_push = 0, c_stale = 0, steps = 0;

    // Every loop decision reads state frozen between two grid barriers: all
    // writers of a phase finish before the barrier that ends it, and nobody
    // writes again until after the barrier that follows the reads (otherwise a
    // fast CTA could change a counter under a slow one and split the grid).
    for (;;) {
        const unsigned long long nn = ld_relaxed_u64(&p.cnt->near_cnt[cur].v);
        const unsigned long long nfar = ld_relaxed_u64(&p.cnt->far_cnt[fcur].v);
        const unsigned st = ld_relaxed_u32(&p.ctl->status);
        grid.sync();
        if (st || (nn == 0 && nfar == 0)) break;
        if (nn == 0) {
            // ---- advance the split and partition the Far pile
            split += p.delta;
            for (unsigned long long i = gtid; i < ((nfar + 31) & ~31ull); i += nthreads) {
                unsigned v = 0;
                unsigned long long d = 0;
                bool live = false;
                if (i < nfar) {
                    NFItem<DistT>::get(p.far[fcur], i, v, d);
                    live = (unsigned long long)__ldcg(p.dist + v) >= d;  // drop stale items
                    c_stale += !live;
                }
                nf_append(p, p.near[cur], &p.cnt->near_cnt[cur], live && d < split, v, d);
                nf_append(p, p.far[fcur ^ 1], &p.cnt->far_cnt[fcur ^ 1], live && d >= split, v, d);
            }
            grid.sync();
            if (gtid == 0) p.cnt->far_cnt[fcur].v = 0;  // read by nobody before the next barrier
            fcur ^= 1;
            continue;
        }
        // ---- one superstep over Near[cur]
        const int nxt = cur ^ 1;
        for (unsigned long long base = gwarp * 32; base < nn; base += nwarps * 32) {
            const unsigned long long i = base + lane;
            unsigned v = 0;
            unsigned long long d = 0, b = 0, e = 0;
            bool live = false;
            if (i < nn) {
                NFItem<DistT>::get(p.near[cur], i, v, d);
                live = (unsigned long long)__ldcg(p.dist + v) >= d;
                if (live) {
                    b = p.off[v];
                    e = p.off[v + 1];
                    ++c_vert;
                    c_edges += e - b;
                } else {
                    ++c_stale;
                }
            }
            // large rows: the whole warp strides over the row (coalesced)
            unsigned big = __ballot_sync(0xffffffffu, live && e - b >= 32);
            while (big) {
                const int src = __ffs(big) - 1;
                big &= big - 1;
                const unsigned long long bb = __shfl_sync(0xffffffffu, b, src), ee = __shfl_sync(0xffffffffu, e, src);
                const unsigned long long dd = __shfl_sync(0xffffffffu, d, src);
                for (unsigned long long a0 = bb; a0 < ee; a0 += 32) {
                    const unsigned long long a = a0 + lane;
                    bool push = false;
                    unsigned t = 0;
                    unsigned long long nd = 0;
                    if (a < ee) {
                        const uint2 arc = p.adj[a];
                        t = arc.x;
                        nd = dd + arc.y;
                        if (nd >= kInf) {
                            atomicOr(&p.ctl->status, kStDistOverflow);
                        } else if (nd < (unsigned long long)__ldcg(p.dist + t)) {
                            push = nd < (unsigned long long)atomicMin(p.dist + t, (DistT)nd);
                        }
                    }
                    c_push += push;
                    nf_append(p, p.near[nxt], &p.cnt->near_cnt[nxt], push && nd < split, t, nd);
                    nf_append(p, p.far[fcur], &p.cnt->far_cnt[fcur], push && nd >= split, t, nd);
                }
            }
            // small rows: each lane walks its own row
            const bool mine = live && e - b < 32;
            const unsigned long long deg = mine ? e - b : 0;
            unsigned long long maxdeg = deg;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) maxdeg = max(maxdeg, __shfl_xor_sync(0xffffffffu, maxdeg, o));
            for (unsigned long long j = 0; j < maxdeg; ++j) {
                bool push = false;
                unsigned t = 0;
                unsigned long long nd = 0;
                if (j < deg) {
                    const uint2 arc = p.adj[b + j];
                    t = arc.x;
                    nd = d + arc.y;
                    if (nd >= kInf) {
                        atomicOr(&p.ctl->status, kStDistOverflow);
                    } else if (nd < (unsigned long long)__ldcg(p.dist + t)) {
                        push = nd < (unsigned long long)atomicMin(p.dist + t, (DistT)nd);
                    }
                }
                c_push += push;
                nf_append(p, p.near[nxt], &p.cnt->near_cnt[nxt], push && nd < split, t, nd);
                nf_append(p, p.far[fcur], &p.cnt->far_cnt[fcur], push && nd >= split, t, nd);
            }
        }
        if (gtid == 0 && globaltimer() - p.ctl->t_start > p.timeout_ns) atomicOr(&p.ctl->status, kStTimeout);
        grid.sync();
        if (gtid == 0) {
            p.cnt->near_cnt[cur].v = 0;  // read by nobody before the next barrier
            ++steps;
        }
        cur = nxt;
    }
    // statistics (warp-reduced, one atomic per warp)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        c_vert += __shfl_xor_sync(0xffffffffu, c_vert, o);
        c_edges += __shfl_xor_sync(0xffffffffu, c_edges, o);
        c_push += __shfl_xor_sync(0xffffffffu, c_push, o);
        c_stale += __shfl_xor_sync(0xffffffffu, c_stale, o);
    }
    if (lane == 0) {
        atomicAdd(&p.ctl->st_vertices, c_vert);
        atomicAdd(&p.ctl->st_edges, c_edges);
        atomicAdd(&p.ctl->st_pushes, c_push);
        atomicAdd(&p.ctl->st_stale, c_stale);
    }
    if (gtid == 0) p.ctl->head_switches = (unsigned)steps;  // reported as supersteps
}

// init: dist = inf, dist[s] = 0, Near[0] = {s}, counters reset
template <typename DistT>
__global__ void near_far_init_kernel(DistT* dist, unsigned n, unsigned source, NFCounters* cnt, Ctl* ctl,
                                     unsigned long long* near0) {
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        dist[v] = (v == source) ? (DistT)0 : DistInf<DistT>::value;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        NFItem<DistT>::put(near0, 0, source, 0ull);
        cnt->near_cnt[0].v = 1;
        cnt->near_cnt[1].v = 0;
        cnt->far_cnt[0].v = 0;
        cnt->far_cnt[1].v = 0;
        cnt->supersteps.v = 0;
        ctl->status = 0;
        ctl->head_switches = 0;
        ctl->delta_changes = 0;
        ctl->trace_count = 0;
        ctl->t_start = globaltimer();
        ctl->st_vertices = ctl->st_edges = ctl->st_pushes = ctl->st_stale = ctl->st_local = 0;
        ctl->reach_v = ctl->reach_e = ctl->max_dist = 0;
        ctl->head.meta = 0;
        for (int i = 0; i < (int)kProfCounters; ++i) ctl->prof[i] = 0;
    }
}

}  // namespace adds

// adds_warp_kernel.cuh -- warp-granular persistent ADDS worker (throughput regime).
//
// Same worklist protocol as adds_persistent_kernel (adds_kernel.cuh): the same
// bucket ring, counters, head CAS, Delta controller, hub-split chunk queue and
// exact quiescence; the difference is the unit of work.  Here every WARP is an
// independent worker with no CTA barrier anywhere:
//
//   claim    (§8(a) A4) claim_batch() by the warp for itself:
//            up to 32 items (one per lane) from the highest-priority active bucket.
//   pop      (A5) lane i loads item i, clears its slot, re-reads dist[v] (stale
//            check) and the row offsets in one round trip.
//   expand   (A5) warp exclusive scan of the 32 degrees (shuffles); lanes take
//            consecutive arcs of the warp's arc space (coalesced 8-byte {col,w}
//            loads, EPT in flight per lane, software-pipelined one round ahead);
//            owners by binary search over the 32-entry scan in shared memory.
//   relax    (A6) nd = d + w, a plain L2 load filters, then atomicMin.
//   push     (A7) improved children are staged in the warp's own
//            shared-memory area (match_any per bucket offset), then flushed with
//            one reserve atomic per (warp flush, bucket) and coalesced ring stores.
//   complete (A8) done += batch.
//
// Why (D12): ncu on the CTA kernel attributes 27-38 % of warp stall
// samples to barriers (warps of a CTA waiting for the slowest slice, or for
// warp 0's claim) on RMAT/ER.  The kernel is bound by random L2 accesses in
// flight, and a warp stalled at a barrier has none; independent warps keep
// issuing.  Hub vertices are split into split_deg-arc chunks (D9) so no warp
// streams a 3.5x10^5-arc row alone.
#pragma once
#include "adds_kernel.cuh"

namespace adds {

template <typename DistT>
struct alignas(16) WarpSmem {
    using Raw = typename ItemT<DistT>::Raw;
    static constexpr int kWS = 256;  // staged pushes per warp (flushed early when full)
    Raw items[kWS];
    unsigned long long ebeg[32];  // row begin of the batch's items
    unsigned long long base[32];  // flush: reserved ring index per bucket offset
    DistT d[32];                  // item distance
    unsigned scan[32];            // exclusive scan of degrees
    unsigned cnt[32];             // staged items per bucket offset
    unsigned short rank[kWS];     // rank of a staged item within its bucket offset
    unsigned char soff[kWS];      // bucket offset of a staged item
};

template <typename DistT, int BT, int EPT, int MINB, bool kF>
__global__ void __launch_bounds__(BT, MINB) adds_warp_kernel(const Params<DistT> p) {
    using IT = ItemT<DistT>;
    using WS = WarpSmem<DistT>;
    constexpr int kWS = WS::kWS;
    constexpr unsigned long long kInf = (unsigned long long)DistInf<DistT>::value;
    constexpr unsigned kChunk = 32u * EPT;

    extern __shared__ __align__(16) unsigned char smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    WS& S = ((WS*)smem)[warp];
    const unsigned lt_mask = lanemask_lt();
    const unsigned nbm = p.nb - 1;
    const unsigned long long pol_stream = policy_evict_first();
    const unsigned long long pol_keep = policy_evict_last(p.keep_frac);
    unsigned long long c_vert = 0, c_edges = 0, c_push = 0, c_stale = 0;  // lane 0
    unsigned backoff = 0;
    S.cnt[lane] = 0;
    __syncwarp();

    for (;;) {
        unsigned slot = 0, st = 0;
        unsigned long long idx = 0;
        Head hd;
        bool is_task = false;
        const unsigned got = claim_batch<DistT, 32>(p, lane, slot, idx, hd, st, is_task);
        if (st) break;
        if (!got) {
            if (try_advance<DistT>(p, hd, lane)) break;
            if (lane == 0) {
                if (globaltimer() - p.ctl->t_start > p.timeout_ns) atomicOr(&p.ctl->status, kStTimeout);
                backoff = backoff ? (backoff * 2 < p.max_backoff_ns ? backoff * 2 : p.max_backoff_ns) : 32;
                __nanosleep(backoff);
            }
            __syncwarp();
            continue;
        }
        backoff = 0;
        const unsigned hs = meta_hs(hd.meta), k = meta_k(hd.meta);

        // ------------------------------------------------------------ pop + stale check
        unsigned deg = 0;
        bool live = false;
        unsigned fword = 0, fbit = 0;
        unsigned long long rb = 0, dv = 0;
        if (is_task) {
            if (lane == 0) {
                SplitTask* tp = p.tasks + (idx & (p.tcap - 1));
                const unsigned len = take_chunk(p, tp);
                if (len) {
                    const unsigned long long b = __ldcg(&tp->beg), d = __ldcg(&tp->d);
                    const unsigned v = __ldcg(&tp->v);
                    slot = __ldcg(&tp->slot);
                    st_release_u32(&tp->len, 0u);
                    const unsigned long long cur = (unsigned long long)ld_keep(p.dist + v, pol_keep);
                    if (cur >= d) {
                        deg = len;
                        rb = b;
                        dv = d;
                        live = true;
                    }
                }
            }
            slot = __shfl_sync(FULL, slot, 0);
        } else if (lane < (int)got) {
            uint32_t v;
            unsigned long long d;
            const unsigned long long ix = (idx + lane) & (p.cap - 1);
            char* sp = p.ring + ((size_t)slot * p.cap + ix) * IT::kBytes;
            unsigned spins = 0;
            bool loaded;
            while (!(loaded = IT::load(sp, v, d)))
                if ((++spins & 1023) == 0 && ld_relaxed_u32(&p.ctl->status)) break;
            if (loaded) {
                IT::clear(sp);  // the slot's one reader this run (D13)
                const unsigned long long cur = (unsigned long long)ld_keep(p.dist + v, pol_keep);
                const unsigned long long b = ld_stream_u64(p.off + v, pol_stream);
                const unsigned long long e = ld_stream_u64(p.off + v + 1, pol_stream);
                if (cur >= d) {
                    deg = (unsigned)(e - b);
                    rb = b;
                    dv = d;
                    live = true;
                    if (p.dynamic) {
                        const unsigned bit = 1u << (v & 31);
                        fword = atomicOr(p.expanded + (v >> 5), bit);
                        fbit = bit;
                    }
                    if (p.split_deg && deg > p.split_deg) deg = spawn_chunks(p, v, d, b, deg, slot);
                }
            }
        }
        unsigned x = deg;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned y = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += y;
        }
        const unsigned E = __shfl_sync(FULL, x, 31);
        S.scan[lane] = x - deg;
        S.ebeg[lane] = rb;
        S.d[lane] = (DistT)dv;
        const unsigned nlive = (unsigned)__popc(__ballot_sync(FULL, live));
        if (lane == 0) {
            if (!is_task) {
                c_vert += nlive;
                c_stale += got - nlive;
            }
            c_edges += E;
        }
        __syncwarp();

        // ------------------------------------------------------------ stream + relax + push
        unsigned s_n = 0;  // staged pushes (warp-uniform)
        auto flush = [&]() {
            __syncwarp();
            const unsigned c = lane < (int)p.nb ? S.cnt[lane] : 0u;
            if (c) {
                const unsigned sl = (hs + lane) & nbm;
                const unsigned long long b = atomicAdd(&p.bk[sl].reserve.v, (unsigned long long)c);
                S.base[lane] = b;
                if (b + c > p.cap) atomicOr(&p.ctl->status, kStRingOverflow);  // no laps (D13)
                if (p.dynamic && lane == (int)nbm) atomicAdd(&p.ctl->g_clip, (unsigned long long)c);
            }
            if (p.dynamic && lane == 0) atomicAdd(&p.ctl->g_push, (unsigned long long)s_n);
            __syncwarp();
            for (unsigned i = lane; i < s_n; i += 32) {
                const unsigned o = S.soff[i];
                const unsigned sl = (hs + o) & nbm;
                const unsigned long long ix = S.base[o] + S.rank[i];
                if (ix < p.cap) IT::store(p.ring + ((size_t)sl * p.cap + ix) * IT::kBytes, S.items[i]);  // D13
            }
            __syncwarp();
            if (c) {
                atomicAdd(&p.bk[(hs + lane) & nbm].avail.v, (unsigned long long)c);  // publish
                S.cnt[lane] = 0;
            }
            if (lane == 0) c_push += s_n;
            s_n = 0;
            __syncwarp();
        };
        auto emit = [&](const bool pg, const unsigned v, const unsigned long long ndv, const unsigned o) {
            const unsigned act = __ballot_sync(FULL, pg);
            if (!act) return;
            const unsigned nact = (unsigned)__popc(act);
            if (s_n + nact > (unsigned)kWS) flush();
            if (pg) {
                const unsigned peers = __match_any_sync(act, o);
                const int pl = __ffs(peers) - 1;
                unsigned r0 = 0;
                if (lane == pl) {
                    r0 = S.cnt[o];
                    S.cnt[o] = r0 + (unsigned)__popc(peers);
                }
                r0 = __shfl_sync(peers, r0, pl) + __popc(peers & lt_mask);
                const unsigned my = s_n + __popc(act & lt_mask);
                S.items[my] = IT::make(v, ndv);
                S.soff[my] = (unsigned char)o;
                S.rank[my] = (unsigned short)r0;
            }
            s_n += nact;
            __syncwarp();
        };
        auto fetch = [&](unsigned base, unsigned (&own)[EPT], uint2 (&a)[EPT]) {
#pragma unroll
            for (int j = 0; j < EPT; ++j) {
                const unsigned e = base + j * 32 + lane;
                unsigned lo = 0, hi = got - 1;
                if (e < E) {
                    while (lo < hi) {
                        const unsigned mid = (lo + hi + 1) >> 1;
                        if (S.scan[mid] <= e) lo = mid;
                        else hi = mid - 1;
                    }
                }
                own[j] = lo;
            }
#pragma unroll
            for (int j = 0; j < EPT; ++j) {
                const unsigned e = base + j * 32 + lane;
                a[j] = e < E ? ld_stream_u2(p.adj + S.ebeg[own[j]] + (e - S.scan[own[j]]), pol_stream)
                             : make_uint2(0u, 0u);
            }
        };
        auto body = [&](const unsigned base, const unsigned (&own)[EPT], const uint2 (&a)[EPT]) {
            unsigned long long nd[EPT];
            DistT cur[EPT];
#pragma unroll
            for (int j = 0; j < EPT; ++j) {
                const unsigned e = base + j * 32 + lane;
                nd[j] = e < E ? relax_sum<kF>((unsigned long long)S.d[own[j]], a[j].y) : kInf;
            }
#pragma unroll
            for (int j = 0; j < EPT; ++j)  // EPT independent L2 gathers in flight
                cur[j] = nd[j] < kInf ? ld_keep(p.dist + a[j].x, pol_keep) : (DistT)0;
            DistT old[EPT];
            bool tried[EPT];
#pragma unroll
            for (int j = 0; j < EPT; ++j) {  // all atomics issued before any result is used
                const unsigned e = base + j * 32 + lane;
                tried[j] = false;
                old[j] = (DistT)0;
                if (e < E) {
                    if (sum_unusable<kF>(nd[j], kInf)) {
                        if (!kF) atomicOr(&p.ctl->status, kStDistOverflow);
                    } else if (nd[j] < (unsigned long long)cur[j]) {
                        old[j] = atomic_min_keep(p.dist + a[j].x, (DistT)nd[j], pol_keep);
                        tried[j] = true;
                    }
                }
            }
#pragma unroll
            for (int j = 0; j < EPT; ++j) {
                const bool push = tried[j] && nd[j] < (unsigned long long)old[j];
                if (!__any_sync(FULL, push)) continue;
                const unsigned o = push ? bucket_of<kF>(nd[j], k, hd.h, p.nb) : 0u;
                emit(push, a[j].x, nd[j], o);
            }
        };
        {
            unsigned own_n[EPT];
            uint2 a_n[EPT];
            if (E > 0) fetch(0, own_n, a_n);
            for (unsigned base = 0; base < E;) {
                unsigned own[EPT];
                uint2 a[EPT];
#pragma unroll
                for (int j = 0; j < EPT; ++j) {
                    own[j] = own_n[j];
                    a[j] = a_n[j];
                }
                const unsigned nxt = base + kChunk;
                if (nxt < E) fetch(nxt, own_n, a_n);  // software pipeline: next round's arcs in flight
                body(base, own, a);
                base = nxt;
            }
        }
        if (s_n) flush();

        // ------------------------------------------------------------ complete
        const unsigned nfirst = (unsigned)__popc(__ballot_sync(FULL, fbit != 0 && (fword & fbit) == 0));
        if (p.dynamic) {
            unsigned run_ctl = 0;
            if (lane == 0) {
                const unsigned nexp = is_task ? 0u : nlive;
                if (nexp) {
                    atomicAdd(&p.ctl->g_exp, (unsigned long long)nexp);
                    atomicAdd(&p.ctl->g_first, (unsigned long long)nfirst);
                }
                const unsigned long long now = globaltimer();
                const unsigned long long last = ld_relaxed_u64(&p.ctl->last_ctl_ns);
                if (now - last > p.period_ns && atomicCAS(&p.ctl->last_ctl_ns, last, now) == last) run_ctl = 1;
            }
            // the children's reserve atomics (returned above) precede the completion
            if (lane == 0) atomicAdd(&p.bk[slot].done.v, (unsigned long long)got);
            if (__shfl_sync(FULL, run_ctl, 0)) periodic_step<DistT>(p, lane);
        } else if (lane == 0) {
            atomicAdd(&p.bk[slot].done.v, (unsigned long long)got);
        }
        __syncwarp();
    }

    if (lane == 0) {
        atomicAdd(&p.ctl->st_vertices, c_vert);
        atomicAdd(&p.ctl->st_edges, c_edges);
        atomicAdd(&p.ctl->st_pushes, c_push);
        atomicAdd(&p.ctl->st_stale, c_stale);
    }
}

}  // namespace adds

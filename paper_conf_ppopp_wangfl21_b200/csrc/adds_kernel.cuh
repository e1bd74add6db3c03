// adds_kernel.cuh -- the persistent ADDS worker kernel for sm_100a.
//
// One launch runs one single-source SSSP to completion.  Every CTA of the grid
// is co-resident (cooperative launch) and loops, with no grid-wide barrier:
//
//   claim    (§8(a) A4)  warp 0 scans the active
//            window of the 32-bucket ring (one lane per bucket), picks the
//            highest-priority bucket with published items and claims a batch
//            through the bucket's avail gate + claim counter (the decentralised
//            replacement of the paper's Manager Thread Block, D1).
//   pop      items are {vertex, distance-at-push}; a slot is empty until its
//            single 64-bit (or 2x64-bit) store lands, so the item's own store is
//            its publication (D2; replaces the WCC segments of P:161).
//            The popper clears the slot behind it.
//   stale    (A5) an item whose vertex already has a smaller distance is skipped.
//   expand   (A5) CTA-cooperative load balancing: exclusive scan of the batch's
//            degrees, then each thread takes consecutive arcs (coalesced
//            interleaved {col,w} loads) and finds its owner by binary search.
//   relax    (A6) nd = d + w; a plain L2 load filters, then atomicMin on
//            dist; the arc improves iff nd < old.
//   push     (A7) improved vertices go to bucket floor(nd/Delta)
//            relative to the head, clipped into the tail.  Warp-aggregated
//            shared-memory staging (ballot + match_any), then one reserve atomic
//            per (CTA flush, bucket) and coalesced stores into the ring.
//   complete (A8) done (= CWC) += batch, outstanding -= batch.
//   advance  (A8/A9) an idle CTA that sees the head bucket
//            complete (done == reserve, acquire-ordered) moves the head to the
//            next non-empty bucket with one 128-bit CAS, running the Delta
//            controller on the ring's occupancy in the same step.
//   finish   (A10) outstanding == 0 <=> no item pushed and unfinished.
#pragma once
#include "bucket_map.h"
#include "common.cuh"

namespace adds {

constexpr unsigned FULL = 0xffffffffu;

template <typename DistT>
struct Params {
    const unsigned long long* __restrict__ off;  // row_offsets[n+1]
    const uint2* __restrict__ adj;               // interleaved {col, w}[m]
    DistT* dist;                                 // n
    char* ring;                                  // nb * cap items
    BucketCtl* bk;                               // nb
    Ctl* ctl;
    TraceEntry* trace;
    unsigned trace_cap;  // 0 = tracing off
    unsigned n;
    unsigned nb;               // ring buckets, power of two <= 32
    unsigned long long cap;    // items per bucket array, power of two
    unsigned dynamic;          // Delta controller enabled
    unsigned clip_pct;         // P:207 (65)
    unsigned settle;           // P:215 head switches between Delta changes
    unsigned util_lo_pct, util_hi_pct;  // P:211 limits, % of resident threads
    unsigned long long resident_threads;
    unsigned avg_deg_x16;      // 16 * m / n  ("correlating ... with the average degree")
    unsigned batch_min;
    unsigned share_shift;      // a CTA claims about avail >> share_shift items
    unsigned k_max;
    unsigned long long timeout_ns;
};

enum { CMD_WORK = 0, CMD_IDLE = 1, CMD_EXIT = 2 };

__device__ __forceinline__ long long warp_sum_s64(long long x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(FULL, x, o);
    return x;
}

// --------------------------------------------------------------- head advance
// Warp-cooperative (lane i <-> ring offset i).  Called by an idle CTA.
template <typename DistT>
__device__ void try_advance(const Params<DistT>& p, const Head hd, const int lane) {
    const unsigned nb = p.nb;
    const unsigned hs = meta_hs(hd.meta), k = meta_k(hd.meta), A = meta_A(hd.meta);
    const unsigned flo = meta_floor(hd.meta), since = meta_since(hd.meta);
    const unsigned slot = (hs + lane) & (nb - 1);
    long long pend = 0;
    if (lane < (int)nb) {
        // done first (acquire), then reserve: done(t1) == reserve(t2) with t1 < t2
        // and done <= reserve at all times  =>  the bucket was complete at t2.
        const unsigned long long d = ld_acquire_u64(&p.bk[slot].done.v);
        const unsigned long long r = ld_relaxed_u64(&p.bk[slot].reserve.v);
        pend = (long long)(r - d);
    }
    const long long head_pend = __shfl_sync(FULL, pend, 0);
    const unsigned nz = __ballot_sync(FULL, lane > 0 && lane < (int)nb && pend > 0);
    if (head_pend != 0 || nz == 0) return;  // head busy, or everything in flight / done
    const unsigned o = __ffs(nz) - 1;       // first non-empty bucket after the head
    const long long total = warp_sum_s64(pend);
    const long long tail = __shfl_sync(FULL, pend, nb - 1);
    const long long win = warp_sum_s64((lane >= (int)o && lane < (int)(o + A)) ? pend : 0);
    if (lane != 0) return;

    unsigned nk = k, nA = A, nflo = flo, nsince = since + 1;
    bool changed = false;
    if (p.dynamic) {
        // utilisation = edge work available in the active window
        const unsigned long long util = ((unsigned long long)win * p.avg_deg_x16) >> 4;
        const unsigned long long T = p.resident_threads;
        const bool low = util * 100ull < (unsigned long long)p.util_lo_pct * T;
        const bool high = util * 100ull > (unsigned long long)p.util_hi_pct * T;
        if (total >= 64 && tail * 100 >= (long long)p.clip_pct * total && nk < p.k_max) {
            nk = k + 1;  // clipping: raise Delta and its lower bound
            nflo = nk;
            changed = true;
        } else if (nsince >= p.settle) {  // settle for K head switches
            if (low && nk < p.k_max) {
                nk = k + 1;
                changed = true;
            } else if (high && nk > nflo) {
                nk = k - 1;
                changed = true;
            }
        }
        if (changed) nsince = 0;
        // fine-grained knob: number of active buckets
        if (low && nA < nb) nA = nA + 1;
        else if (high && nA > 1) nA = nA - 1;
    }
    unsigned long long nh = hd.h + o;
    if (nk > k) nh >>= (nk - k);
    else if (nk < k) nh <<= (k - nk);
    const Head nhd{nh, pack_meta((hs + o) & (nb - 1), nk, nA, nflo, nsince > 0xffff ? 0xffff : nsince)};
    Head seen;
    if (cas_head(&p.ctl->head, hd, nhd, seen)) {
        atomicAdd(&p.ctl->head_switches, 1u);
        if (nk != k) atomicAdd(&p.ctl->delta_changes, 1u);
        if (p.trace_cap) {
            const unsigned t = atomicAdd(&p.ctl->trace_count, 1u);
            if (t < p.trace_cap) {
                TraceEntry e;
                e.time_ns = globaltimer();
                e.head = nh;
                e.pending_total = (unsigned long long)total;
                e.pending_window = (unsigned long long)win;
                e.pending_tail = (unsigned long long)tail;
                e.delta_log2 = nk;
                e.active = nA;
                p.trace[t] = e;
            }
        }
    }
}

// --------------------------------------------------------------- kernel
template <typename DistT, int BT>
__global__ void __launch_bounds__(BT) adds_persistent_kernel(const Params<DistT> p) {
    using IT = ItemT<DistT>;
    using Raw = typename IT::Raw;
    constexpr int kStage = 2 * BT;  // staged pushes before a forced flush
    constexpr int kWarps = BT / 32;
    constexpr unsigned long long kInf = (unsigned long long)DistInf<DistT>::value;

    __shared__ Raw s_items[kStage];
    __shared__ unsigned char s_soff[kStage];
    __shared__ unsigned short s_rank[kStage];
    __shared__ unsigned s_cnt[kMaxBuckets];
    __shared__ unsigned long long s_base[kMaxBuckets];
    __shared__ unsigned long long s_ebeg[BT];
    __shared__ DistT s_d[BT];
    __shared__ unsigned s_scan[BT];
    __shared__ unsigned s_wsum[kWarps];
    __shared__ unsigned s_total, s_E, s_got, s_slot;
    __shared__ int s_cmd;
    __shared__ unsigned long long s_idx;
    __shared__ Head s_head;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const unsigned nbm = p.nb - 1;
    unsigned long long c_vert = 0, c_edges = 0, c_push = 0, c_stale = 0;  // thread 0
    unsigned backoff = 0;

    if (tid < (int)kMaxBuckets) s_cnt[tid] = 0;
    if (tid == 0) s_total = 0;
    __syncthreads();

    for (;;) {
        // ------------------------------------------------------------ claim
        if (warp == 0) {
            int cmd = CMD_IDLE;
            unsigned st = 0;
            if (lane == 0) st = ld_relaxed_u32(&p.ctl->status);
            st = __shfl_sync(FULL, st, 0);
            if (st) {
                cmd = CMD_EXIT;
            } else {
                const Head hd = ld_head(&p.ctl->head);
                const unsigned hs = meta_hs(hd.meta), A = meta_A(hd.meta);
                const unsigned slot = (hs + lane) & nbm;
                long long av = 0;
                if (lane < (int)A) av = (long long)ld_relaxed_u64(&p.bk[slot].avail.v);
                unsigned mask = __ballot_sync(FULL, av > 0);
                while (mask) {  // higher-priority buckets first
                    const int f = __ffs(mask) - 1;
                    unsigned got = 0;
                    if (lane == f) {
                        long long want = av >> p.share_shift;
                        if (want < (long long)p.batch_min) want = p.batch_min;
                        if (want > BT) want = BT;
                        unsigned long long* avp = &p.bk[slot].avail.v;
                        const long long old = (long long)atomicAdd(avp, (unsigned long long)(-want));
                        const long long g = old <= 0 ? 0 : (old < want ? old : want);
                        if (g < want) atomicAdd(avp, (unsigned long long)(want - g));
                        if (g > 0) {
                            s_idx = atomicAdd(&p.bk[slot].claim.v, (unsigned long long)g);
                            s_got = (unsigned)g;
                            s_slot = slot;
                            s_head = hd;
                        }
                        got = (unsigned)g;
                    }
                    got = __shfl_sync(FULL, got, f);
                    if (got) {
                        cmd = CMD_WORK;
                        break;
                    }
                    mask &= mask - 1;
                }
                if (cmd != CMD_WORK) {
                    long long out = 0;
                    if (lane == 0) out = ld_relaxed_s64(&p.ctl->outstanding);
                    out = __shfl_sync(FULL, out, 0);
                    if (out == 0) {
                        cmd = CMD_EXIT;
                    } else {
                        try_advance<DistT>(p, hd, lane);
                        if (lane == 0) {
                            if (globaltimer() - p.ctl->t_start > p.timeout_ns) atomicOr(&p.ctl->status, kStTimeout);
                            backoff = backoff ? (backoff < 512 ? backoff * 2 : 1024) : 32;
                            __nanosleep(backoff);
                        }
                    }
                } else if (lane == 0) {
                    backoff = 0;
                }
            }
            if (lane == 0) s_cmd = cmd;
        }
        __syncthreads();
        const int cmd = s_cmd;
        if (cmd == CMD_EXIT) break;
        if (cmd == CMD_IDLE) continue;

        // ------------------------------------------------------------ pop + stale check
        const unsigned got = s_got, slot = s_slot;
        const Head hd = s_head;
        const unsigned hs = meta_hs(hd.meta), k = meta_k(hd.meta);
        unsigned deg = 0;
        bool live = false;
        if (tid < (int)got) {
            const unsigned long long idx = (s_idx + tid) & (p.cap - 1);
            char* sp = p.ring + ((size_t)slot * p.cap + idx) * IT::kBytes;
            uint32_t v;
            unsigned long long d;
            unsigned spins = 0;
            bool loaded;
            while (!(loaded = IT::load(sp, v, d))) {  // reserved, store not landed yet
                if ((++spins & 1023) == 0 && ld_relaxed_u32(&p.ctl->status)) break;  // aborted run
            }
            if (loaded) {
                IT::clear(sp);
                const unsigned long long cur = (unsigned long long)ld_cg(p.dist + v);
                if (cur >= d) {  // not stale: d is still v's distance ("refined")
                    const unsigned long long b = p.off[v], e = p.off[v + 1];
                    deg = (unsigned)(e - b);
                    s_ebeg[tid] = b;
                    s_d[tid] = (DistT)d;
                    live = true;
                }
            }
        }
        // exclusive scan of degrees over the CTA
        unsigned x = deg;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned y = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) s_wsum[warp] = x;
        const int nlive = __syncthreads_count(live);
        if (warp == 0) {
            const unsigned ws = lane < kWarps ? s_wsum[lane] : 0;
            unsigned inc = ws;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned y = __shfl_up_sync(FULL, inc, o);
                if (lane >= o) inc += y;
            }
            if (lane < kWarps) s_wsum[lane] = inc - ws;
            if (lane == kWarps - 1) s_E = inc;
        }
        __syncthreads();
        s_scan[tid] = x - deg + s_wsum[warp];
        const unsigned E = s_E;
        __syncthreads();
        if (tid == 0) {
            c_vert += nlive;
            c_stale += got - nlive;
            c_edges += E;
        }

        // ------------------------------------------------------------ expand + relax + push
        for (unsigned base = 0; base < E; base += BT) {
            const unsigned e = base + tid;
            bool push = false;
            uint32_t pv = 0;
            unsigned long long pd = 0;
            if (e < E) {
                unsigned lo = 0, hi = got - 1;  // owner = largest i with scan[i] <= e
                while (lo < hi) {
                    const unsigned mid = (lo + hi + 1) >> 1;
                    if (s_scan[mid] <= e) lo = mid;
                    else hi = mid - 1;
                }
                const uint2 a = __ldg(p.adj + s_ebeg[lo] + (e - s_scan[lo]));
                const unsigned long long nd = (unsigned long long)s_d[lo] + a.y;
                if (nd >= kInf) {
                    atomicOr(&p.ctl->status, kStDistOverflow);  // 32-bit distances insufficient
                } else {
                    const DistT cur = ld_cg(p.dist + a.x);
                    if (nd < (unsigned long long)cur) {
                        const DistT old = atomicMin(p.dist + a.x, (DistT)nd);
                        if (nd < (unsigned long long)old) {
                            push = true;
                            pv = a.x;
                            pd = nd;
                        }
                    }
                }
            }
            // warp-aggregated staging: one smem atomic per warp for the slot, one
            // per (warp, bucket) for the rank inside the bucket's run
            const unsigned act = __ballot_sync(FULL, push);
            if (push) {
                const unsigned o = adds_bucket_offset(pd, k, hd.h, p.nb);
                const int leader = __ffs(act) - 1;
                unsigned pos = 0;
                if (lane == leader) pos = atomicAdd(&s_total, (unsigned)__popc(act));
                pos = __shfl_sync(act, pos, leader) + __popc(act & lanemask_lt());
                const unsigned peers = __match_any_sync(act, o);
                const int pl = __ffs(peers) - 1;
                unsigned r0 = 0;
                if (lane == pl) r0 = atomicAdd(&s_cnt[o], (unsigned)__popc(peers));
                r0 = __shfl_sync(peers, r0, pl) + __popc(peers & lanemask_lt());
                s_items[pos] = IT::make(pv, pd);
                s_soff[pos] = (unsigned char)o;
                s_rank[pos] = (unsigned short)r0;
            }
            __syncthreads();
            const unsigned total = s_total;
            if (total > (unsigned)(kStage - BT) || (base + BT >= E && total > 0)) {
                // ---------------------------------------------------- flush
                if (warp == 0) {
                    if (lane == 0) {
                        // count children before they become claimable (termination);
                        // the returned value is consumed, so the add is performed
                        // before this warp issues the reserves below
                        const long long before =
                            (long long)atomicAdd((unsigned long long*)&p.ctl->outstanding, (unsigned long long)total);
                        if (before <= 0) atomicOr(&p.ctl->status, kStBug);
                        c_push += total;
                    }
                    __syncwarp();
                    if (lane < (int)p.nb) {
                        const unsigned c = s_cnt[lane];
                        if (c) {
                            const unsigned sl = (hs + lane) & nbm;
                            const unsigned long long b = atomicAdd(&p.bk[sl].reserve.v, (unsigned long long)c);
                            s_base[lane] = b;
                            if (b + c > p.cap) {  // lapping: previous occupants must be claimed
                                const unsigned long long cl = ld_relaxed_u64(&p.bk[sl].claim.v);
                                if (b + c - p.cap > cl) atomicOr(&p.ctl->status, kStRingOverflow);
                            }
                        }
                    }
                }
                __syncthreads();
                for (unsigned i = tid; i < total; i += BT) {
                    const unsigned o = s_soff[i];
                    const unsigned sl = (hs + o) & nbm;
                    const unsigned long long idx = s_base[o] + s_rank[i];
                    char* sp = p.ring + ((size_t)sl * p.cap + (idx & (p.cap - 1))) * IT::kBytes;
                    bool ok = true;
                    if (idx >= p.cap) {  // wait for the previous lap's reader to clear it
                        unsigned spins = 0;
                        while (!IT::empty(sp)) {
                            if ((++spins & 255) == 0 && ld_relaxed_u32(&p.ctl->status)) {
                                ok = false;
                                break;
                            }
                        }
                    }
                    if (ok) IT::store(sp, s_items[i]);
                }
                __syncthreads();
                if (warp == 0 && lane < (int)p.nb) {
                    const unsigned c = s_cnt[lane];
                    if (c) {
                        atomicAdd(&p.bk[(hs + lane) & nbm].avail.v, (unsigned long long)c);  // publish
                        s_cnt[lane] = 0;
                    }
                }
                if (tid == 0) s_total = 0;
                __syncthreads();
            }
        }

        // ------------------------------------------------------------ complete
        if (tid == 0) {
            atomicAdd(&p.bk[slot].done.v, (unsigned long long)got);  // CWC
            atomicAdd((unsigned long long*)&p.ctl->outstanding, (unsigned long long)(-(long long)got));
        }
        __syncthreads();
    }

    if (tid == 0) {
        atomicAdd(&p.ctl->st_vertices, c_vert);
        atomicAdd(&p.ctl->st_edges, c_edges);
        atomicAdd(&p.ctl->st_pushes, c_push);
        atomicAdd(&p.ctl->st_stale, c_stale);
    }
}

}  // namespace adds

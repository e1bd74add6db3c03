// adds_kernel.cuh -- the persistent ADDS worker kernel for sm_100a.
//
// One launch runs one single-source SSSP to completion.  Every CTA of the grid
// is co-resident (cooperative launch) and loops, with no grid-wide barrier:
//
//   claim    (§8(a) A4)  warp 0 reads the status,
//            the head state and all 32 buckets' avail gates in ONE round trip
//            (one lane per bucket), picks the highest-priority active bucket
//            with published items and claims a batch (avail gate, then the
//            claim counter = read_ptr).  This decentralises the paper's
//            Manager Thread Block (D1).
//   pop      items are {vertex, distance-at-push}; a ring slot is empty until
//            its single 64-bit (2x64-bit) store lands, so the item's own store
//            is its publication (D2, replaces the WCC segments of
//            P:161).  The popper clears the slot behind it.
//   stale    (A5) an item whose vertex already holds a smaller distance is
//            skipped (checked in parallel with the row-offset loads).
//   expand   (A5) CTA-cooperative load balancing: exclusive scan of the batch's
//            degrees; each thread takes EPT arcs per round (coalesced 8-byte
//            {col,w} loads, EPT loads in flight) and finds their owners by
//            binary search over the scan.
//   relax    (A6) nd = d + w; a plain L2 load filters, then atomicMin on
//            dist; the arc improves iff nd < old.
//   push     (A7) improved vertices go to bucket floor(nd/Delta)
//            relative to the head, clipped into the tail.  Children that land in
//            the head bucket are kept in shared memory and become this CTA's
//            next batch (no ring round trip on the dependency chain, DESIGN.md
//            D3); the rest are staged with warp-aggregated shared-memory
//            atomics (ballot + match_any), reserved with one atomic per (CTA
//            flush, bucket) and stored coalesced.
//   complete (A8) one atomic: done (= CWC) += batch - kept, or
//            local += kept - batch.
//   advance  (A8/A9) an idle CTA that sees the head bucket
//            complete (done == reserve + local, acquire-ordered) moves the head
//            to the next non-empty bucket with one 128-bit CAS and runs the
//            Delta controller on the ring occupancy in the same step.
//   finish   (A10) every bucket complete  <=>  quiescent.
#pragma once
#ifndef STAGE_MULT
#define STAGE_MULT 4  // staging capacity = STAGE_MULT/2 * BT * EPT items
#endif
#include "bucket_map.h"
#include "common.cuh"

namespace adds {

constexpr unsigned FULL = 0xffffffffu;

template <typename DistT>
struct Params {
    const unsigned long long* __restrict__ off;  // row_offsets[n+1]
    const uint2* __restrict__ adj;               // interleaved {col, w}[m]
    const uint2* __restrict__ rows;              // {row begin, degree}[n] when m < 2^32 (else nullptr)
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
    unsigned adapt_active;     // controller varies the active-bucket count in [a_min, a_max]
    unsigned a_min, a_max;
    unsigned grid;             // CTAs of this launch (utilisation = CTAs holding a batch)
    unsigned clip_pct;         // P:207 (65)
    unsigned settle;           // P:215 head switches between Delta changes
    unsigned util_lo_pct, util_hi_pct;  // P:211 limits, % of resident threads
    unsigned long long resident_threads;
    unsigned avg_deg_x16;      // 16 * m / n  ("correlating ... with the average degree")
    unsigned batch_min;
    unsigned share_shift;      // a CTA claims about avail >> share_shift items
    unsigned local_max;        // head-bucket children a CTA keeps for itself (0 = off)
    unsigned warp_local;       // warp-local continuation in the latency regime (0 = off)
    unsigned short* filt;      // n x u16 upper bounds of dist in units of 2^filt_shift (nullptr = off)
    unsigned filt_shift;
    unsigned max_backoff_ns;
    unsigned prof;             // SSSP_FLAG_PROFILE: accumulate per-phase cycles
    float keep_frac;           // fraction of dist covered by the L2 persisting set-aside
    unsigned* expanded;        // n-bit bitmap: vertex expanded at least once (controller waste signal)
    unsigned waste_lo, waste_hi;  // permille
    unsigned long long period_ns;
    unsigned long long startup_first;  // no Delta growth before this many first expansions
    SplitTask* tasks;          // hub-split chunk queue (counters in bk[kSplitQ])
    unsigned long long tcap;   // entries, power of two
    unsigned split_deg;        // split vertices with more arcs than this (0 = off)
    // chunked bucket storage (0 = one no-lap array of cap items per bucket, D13)
    unsigned chunked;
    unsigned* ctab;            // nb x (tab_mask + 1): chunk id + 1 (0 = not taken yet)
    unsigned tab_mask;
    unsigned* chunk_used;      // items read per chunk
    unsigned* free_ring;       // pool_chunks entries: chunk id + 1 (0 = empty)
    ChunkPool* pool;
    unsigned pool_chunks;      // power of two
    unsigned k_max;
    unsigned long long timeout_ns;
};

enum { CMD_WORK = 0, CMD_IDLE = 1, CMD_EXIT = 2 };

__device__ __forceinline__ long long warp_sum_s64(long long x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(FULL, x, o);
    return x;
}

// --------------------------------------------------------------- Delta controller
// P:205-217 (§5.5).  Inputs, read warp-cooperatively (lane i <-> ring offset i):
// pending items per bucket (reserved + kept - done), hence the head, the active
// window (utilisation = window items x average degree vs resident threads,
// P:211) and the tail (clip share); plus the recent re-expansion
// share of expansions (work-waste signal, R6).  Readings:
//   clip   tail >= clip_pct of all pending (2 steps apart) -> Delta x2, floor = Delta
//   waste  share > waste_hi after settling        -> Delta /2 (not below floor)
//   grow   window under-utilised AND share < lo   -> Delta x2
//   A      active buckets follow the same two signals one step at a time
// Settling: `since` counts controller steps (head switches and periodic
// steps) since the last Delta change; a change needs since >= settle (a quarter
// of that for growth while the re-expansion share is below waste_lo / 8).
struct CtlDecision {
    unsigned k, A, flo, since, ceil, pk;
    bool changed;
    unsigned flags;  // decision inputs, recorded in the trace: 1 low, 2 high, 4 beyond, 8 wasteful,
                     // 16 frugal, 32 clipping, 64 waste known, 128 progressed, 256 settled
};

// ratio_x100 = 100 * expansions / distinct vertices expanded so far (cumulative,
// >= 100; 100 = Dijkstra's vertex work).  waste = re-expansion share (permille)
// over the recent window.  clip = share of recent pushes that were clipped.
template <typename DistT>
__device__ CtlDecision decide(const Params<DistT>& p, unsigned k, unsigned A, unsigned flo, unsigned since,
                              unsigned ceil, unsigned pk, bool head_switch, long long total, long long tail, long long win,
                              unsigned waste,
                              bool waste_known, unsigned clip, bool clip_known, unsigned ratio_x100,
                              bool progressed, long long busy) {
    // since = [0,8) controller steps, [8,16) head switches since the last change
    unsigned steps = since & 0xffu, hsw = (since >> 8) & 0xffu;
    steps = steps < 255u ? steps + 1 : 255u;
    if (head_switch && hsw < 255u) ++hsw;
    CtlDecision d{k, A, flo, steps | (hsw << 8), ceil, head_switch ? 0u : pk, false, 0u};
    if (!p.dynamic) return d;
    // the waste ceiling (hysteresis, below) holds for the rest of the run: letting it expire
    // after 64 or 16 head switches regrew ROAD into wasteful Deltas (work 1.63x -> 2.0x,
    // 43.9 -> 47 ms, sweeps §24)
    const unsigned long long util = ((unsigned long long)(win > 0 ? win : 0) * p.avg_deg_x16) >> 4;
    const unsigned long long T = p.resident_threads;
    const bool low = util * 100ull < (unsigned long long)p.util_lo_pct * T;
    const bool high = util * 100ull > (unsigned long long)p.util_hi_pct * T;
    const bool beyond = (total - win) > win;  // more work waits outside the active window
    // waste: recent re-expansions high AND the run as a whole already above 2x
    // (both need the start-up gate: early samples are tiny and noisy)
    const bool wasteful = progressed && waste_known && waste > p.waste_hi && ratio_x100 > 200;
    // frugal: recent re-expansion low, and either the run as a whole is below 1.5x
    // or the recent share is below half the growth limit (a bad start-up must not
    // block growth for the rest of the run)
    // (an unmeasurable waste -- too few expansions in the window -- means the run
    // is crawling: growth is allowed once the start-up gate is open)
    // cumulative-ratio gate on growth: 2.5x Dijkstra's vertex work (road-like graphs sit
    // at 1.6-1.7x at their time-optimal Delta; a 1.5x gate pinned them one step below it,
    // profiles/r01_sweeps.md §19)
    constexpr unsigned ratio_gate = 250u;
    const bool frugal = (!waste_known || waste < p.waste_lo) &&
                        (ratio_x100 < ratio_gate || !waste_known || waste * 2 < p.waste_lo) && progressed;
    // the paper's rule -- the tail holds >= 65 % of the pending items -- applied to
    // live clipping: recent pushes must still be landing in the tail (>= 10 %) and enough work
    // must be pending to matter.  On its own the push share fired on the large tentative
    // distances early in a run (ER grown from its best Delta 2^15 to 2^16, work 1.01x -> 1.17x)
    // and the pending share on a drained ring whose last items sat in the tail slot (ER with
    // degree 4 doubled Delta from 2^21 to 2^31 in its drain; profiles/r02_sweeps.md §5, §7)
    const bool clipping = total >= 1024 && tail * 100 >= (long long)p.clip_pct * total && clip_known && clip >= 100;
    // settled: enough steps AND the head has switched twice since the last
    // change, so the ring has turned over and the items placed under the previous
    // Delta -- whose slots now mix priorities -- are no longer what the
    // waste signal measures (without this, shrinks fed on their own mixing waste)
    const bool turned = hsw >= 2;
    d.flags = (low ? 1u : 0u) | (high ? 2u : 0u) | (beyond ? 4u : 0u) | (wasteful ? 8u : 0u) |
              (frugal ? 16u : 0u) | (clipping ? 32u : 0u) | (waste_known ? 64u : 0u) | (progressed ? 128u : 0u) |
              (steps >= p.settle && turned ? 256u : 0u);
    if (clipping && k < p.k_max && steps >= 2) {
        d.k = k + 1;  // clipping: raise Delta and its lower bound
        d.flo = d.k;
        if (d.ceil <= d.k) d.ceil = 0xffu;  // the clip bound overrides the waste ceiling
        d.changed = true;
    } else if (wasteful && k > flo && steps >= 4 * p.settle && hsw == 0 && d.pk < 2u) {
        // sustained waste while the head does not move (one bucket holding the whole frontier:
        // RMAT with U[1,2^20] re-expanded 6x at 2^15 with the head parked for 20 ms): shrink
        // after four settling periods even without head switches -- at most twice before the
        // head moves again (a correction wave runs on whatever Delta: ROAD collapsed 2^11 -> 2^2
        // this way, every step reading 100 % re-expansions, and then crawled; r02 §12)
        d.k = k - 1;
        d.ceil = k;
        d.pk = d.pk + 1u;
        d.changed = true;
    } else if (steps >= p.settle && turned) {
        if (wasteful && k > flo) {
            d.k = k - 1;
            d.ceil = k;  // hysteresis: do not grow back into a Delta measured wasteful
            d.changed = true;
        } else if (low && frugal && beyond && k < p.k_max && k + 1 < ceil) {
            d.k = k + 1;
            d.changed = true;
        }
    } else if (steps * 4 >= p.settle && turned && low && frugal && beyond && (!waste_known || waste * 8 < p.waste_lo) &&
               k < p.k_max && k + 1 < ceil) {
        d.k = k + 1;  // essentially no re-expansion yet: grow with a quarter of the settling time
        d.changed = true;
    }
    if (d.changed) d.since = 0;
    // fine-grained knob: utilisation as the paper measures it -- the work
    // assigned, here the CTAs holding a batch.  One more active bucket while CTAs are idle,
    // work waits beyond the window and re-expansion is low; one fewer when every CTA is
    // busy or the run is wasteful.  Bounded to [a_min, a_max] around the degree-based
    // default (a wider window on road-like graphs fed the Delta shrink spiral, sweeps r01 §26)
    if (p.adapt_active) {
        const bool idle_ctas = busy * 10 < (long long)p.grid * 9;
        const bool all_busy = busy >= (long long)p.grid;
        if (idle_ctas && beyond && frugal && A < p.a_max)
            d.A = A + 1;
        else if ((wasteful || all_busy) && A > p.a_min)
            d.A = A - 1;
    }
    return d;
}

// Pending items of the 32 buckets relative to the head (acquire-ordered so that a
// zero really means complete): every done is read before any reserve/local.
template <typename DistT>
__device__ __forceinline__ long long bucket_pending(const Params<DistT>& p, unsigned hs, int lane) {
    const unsigned slot = (hs + lane) & (p.nb - 1);
    unsigned long long d = 0, r = 0, l = 0;
    if (lane < (int)p.nb) d = ld_acquire_u64(&p.bk[slot].done.v);
    __syncwarp();
    if (lane < (int)p.nb) {
        r = ld_relaxed_u64(&p.bk[slot].reserve.v);
        l = ld_relaxed_u64(&p.bk[slot].local.v);
    }
    return (long long)(r + l - d);
}

// Re-expansion share of the recent window.  A window too small to measure (a crawling run
// or a drain) keeps the last measured share: an unmeasurable window must not read as
// "no waste" once the run has shown waste (ER with degree 4 grew Delta 2^21 -> 2^25 in its
// drain on such readings, profiles/r02_sweeps.md §7); before any measurement it is unknown.
template <typename DistT>
__device__ __forceinline__ unsigned recent_waste(const Params<DistT>& p, bool& known) {
    const unsigned long long e = ld_relaxed_u64(&p.ctl->g_exp) - ld_relaxed_u64(&p.ctl->exp_mark);
    const unsigned long long f = ld_relaxed_u64(&p.ctl->g_first) - ld_relaxed_u64(&p.ctl->first_mark);
    if (e >= 4096) {
        known = true;
        const unsigned w = e > f ? (unsigned)((e - f) * 1000ull / e) : 0u;
        st_relaxed_u32(&p.ctl->last_waste, w + 1u);
        return w;
    }
    const unsigned lw = ld_relaxed_u32(&p.ctl->last_waste);
    known = lw != 0u;
    return known ? lw - 1u : 0u;
}
template <typename DistT>
__device__ __forceinline__ unsigned cumulative_ratio(const Params<DistT>& p) {
    const unsigned long long e = ld_relaxed_u64(&p.ctl->g_exp), f = ld_relaxed_u64(&p.ctl->g_first);
    return f >= 4096 ? (unsigned)(e * 100ull / f) : 100u;
}
template <typename DistT>
__device__ __forceinline__ unsigned recent_clip(const Params<DistT>& p, bool& known) {
    const unsigned long long q = ld_relaxed_u64(&p.ctl->g_push) - ld_relaxed_u64(&p.ctl->push_mark);
    const unsigned long long c = ld_relaxed_u64(&p.ctl->g_clip) - ld_relaxed_u64(&p.ctl->clip_mark);
    known = q >= 65536;  // a statistically meaningful sample of the push distribution
    return known ? (unsigned)(c * 1000ull / q) : 0u;
}

// Commit a controller step by 128-bit CAS; restart the measurement windows on a
// change and whenever they are full, so the signals track the recent past.
template <typename DistT>
__device__ void commit_step(const Params<DistT>& p, const Head hd, const Head nhd, bool kchanged, unsigned since,
                            long long total, long long win, long long tail, unsigned waste, unsigned reason,
                            unsigned flags, unsigned clip, bool clip_known) {
    Head seen;
    if (!cas_head(&p.ctl->head, hd, nhd, seen)) return;
    if (reason == 1) atomicAdd(&p.ctl->head_switches, 1u);
    if (kchanged) atomicAdd(&p.ctl->delta_changes, 1u);
    // measurement windows are sized in events, not steps: restart after a Delta
    // change, or once a window holds 64K expansions / 256K pushes
    const unsigned long long ge = ld_relaxed_u64(&p.ctl->g_exp), gp = ld_relaxed_u64(&p.ctl->g_push);
    if (kchanged || ge - ld_relaxed_u64(&p.ctl->exp_mark) >= 65536) {
        p.ctl->exp_mark = ge;
        p.ctl->first_mark = ld_relaxed_u64(&p.ctl->g_first);
    }
    if (kchanged || gp - ld_relaxed_u64(&p.ctl->push_mark) >= 262144) {
        p.ctl->push_mark = gp;
        p.ctl->clip_mark = ld_relaxed_u64(&p.ctl->g_clip);
    }
    if (p.trace_cap) {
        const unsigned t = atomicAdd(&p.ctl->trace_count, 1u);
        if (t < p.trace_cap) {
            TraceEntry e;
            e.time_ns = globaltimer();
            e.head = nhd.h;
            e.pending_total = (unsigned long long)total;
            e.pending_window = (unsigned long long)win;
            e.pending_tail = (unsigned long long)tail;
            e.delta_log2 = meta_k(nhd.meta);
            e.active = meta_A(nhd.meta) | (meta_floor(nhd.meta) << 8) | (meta_ceil(nhd.meta) << 16);
            e.waste_permille = waste;
            e.reason = reason | ((flags & 0x1ffu) << 8) | ((clip < 1000u ? clip : 1000u) << 20) |
                       (clip_known ? 1u << 30 : 0u);
            p.trace[t] = e;
        }
    }
}

// Re-express the absolute head bucket number under a new Delta exponent.
__device__ __forceinline__ unsigned long long rehead(unsigned long long h, unsigned k, unsigned nk) {
    if (nk > k) return h >> (nk - k);
    if (nk < k) return h << (k - nk);
    return h;
}

// --------------------------------------------------------------- head advance / termination
// Called by an idle CTA's warp 0.  Returns true when the whole run is quiescent.
template <typename DistT>
__device__ bool try_advance(const Params<DistT>& p, const Head hd, const int lane) {
    const unsigned nb = p.nb;
    const unsigned hs = meta_hs(hd.meta), k = meta_k(hd.meta), A = meta_A(hd.meta);
    // cheap test first: while the head bucket has work in flight there is neither
    // an advance nor termination to detect (one lane, one round trip)
    long long hp = 0;
    if (lane == 0) {
        const unsigned long long d0 = ld_acquire_u64(&p.bk[hs].done.v);
        hp = (long long)(ld_relaxed_u64(&p.bk[hs].reserve.v) + ld_relaxed_u64(&p.bk[hs].local.v) - d0);
    }
    if (__shfl_sync(FULL, hp, 0) != 0) return false;
    const long long pend = bucket_pending(p, hs, lane);
    const long long total = warp_sum_s64(pend);
    if (total == 0) return true;  // every bucket complete: quiescent (reading R11)
    const long long head_pend = __shfl_sync(FULL, pend, 0);
    const unsigned nz = __ballot_sync(FULL, lane > 0 && lane < (int)nb && pend > 0);
    if (head_pend != 0 || nz == 0) return false;  // head busy, or only in-flight work left
    const unsigned o = __ffs(nz) - 1;              // first non-empty bucket after the head
    const long long tail = __shfl_sync(FULL, pend, nb - 1);
    const long long win = warp_sum_s64((lane >= (int)o && lane < (int)(o + A)) ? pend : 0);
    if (lane != 0) return false;
    bool known, cknown;
    const unsigned waste = recent_waste(p, known);
    const unsigned clip = recent_clip(p, cknown);
    const CtlDecision d = decide(p, k, A, meta_floor(hd.meta), meta_since(hd.meta), meta_ceil(hd.meta), meta_pk(hd.meta), true,
                                 total, tail, win, waste,
                                 known, clip, cknown, cumulative_ratio(p),
                                 ld_relaxed_u64(&p.ctl->g_exp) >= p.startup_first ||
                                     ld_relaxed_u32(&p.ctl->head_switches) >= 32u,
                                 (long long)ld_relaxed_u64(&p.ctl->g_busy));
    const Head nhd{rehead(hd.h + o, k, d.k),
                   pack_meta((hs + o) & (nb - 1), d.k, d.A, d.flo, d.since, d.ceil, d.pk)};
    SSSP_FUZZ_AT(FZ_HEAD);
    commit_step(p, hd, nhd, d.k != k, d.since, total, win, tail, waste, 1u, d.flags, clip, cknown);
    return false;
}

// Periodic controller step ("the MTB periodically gathers run-time
// information"), run by warp 0 of a CTA that won the period.  The head stays
// where it is; only its number is re-expressed if Delta changes.
template <typename DistT>
__device__ void periodic_step(const Params<DistT>& p, const int lane) {
    const Head hd = ld_head(&p.ctl->head);
    const unsigned hs = meta_hs(hd.meta), k = meta_k(hd.meta), A = meta_A(hd.meta);
    const long long pend = bucket_pending(p, hs, lane);
    const long long total = warp_sum_s64(pend);
    const long long tail = __shfl_sync(FULL, pend, p.nb - 1);
    const long long win = warp_sum_s64(lane < (int)A ? pend : 0);
    if (lane != 0 || total == 0) return;
    bool known, cknown;
    const unsigned waste = recent_waste(p, known);
    const unsigned clip = recent_clip(p, cknown);
    const CtlDecision d = decide(p, k, A, meta_floor(hd.meta), meta_since(hd.meta), meta_ceil(hd.meta), meta_pk(hd.meta), false,
                                 total, tail, win, waste,
                                 known, clip, cknown, cumulative_ratio(p),
                                 ld_relaxed_u64(&p.ctl->g_exp) >= p.startup_first ||
                                     ld_relaxed_u32(&p.ctl->head_switches) >= 32u,
                                 (long long)ld_relaxed_u64(&p.ctl->g_busy));
    const Head nhd{rehead(hd.h, k, d.k), pack_meta(hs, d.k, d.A, d.flo, d.since, d.ceil, d.pk)};
    commit_step(p, hd, nhd, d.k != k, d.since, total, win, tail, waste, 2u, d.flags, clip, cknown);
}

// --------------------------------------------------------------- weight arithmetic
// Integer weights: nd = d + w in 64 bits, Delta = 2^k, bucket = nd >> k.
// Float32 weights (NEXT-3): d and w are IEEE binary32 bit patterns (non-negative
// floats order like their bits, so dist keeps the native u32 atomicMin);
// nd = fl(d + w) round-to-nearest; Delta = 2^(k - kFloatBias), k biased so that
// Delta can be below 1.
constexpr int kFloatBias = 64;
template <bool kF>
__device__ __forceinline__ unsigned long long relax_sum(unsigned long long d, unsigned w) {
    if constexpr (kF)
        return (unsigned long long)__float_as_uint(__fadd_rn(__uint_as_float((unsigned)d), __uint_as_float(w)));
    else
        return d + w;
}
// a sum that can never be an improvement (float: +inf / NaN) or that overflows
// the distance type (integer: re-run with 64-bit distances)
// The same sum in the distance type's width.  bad = the sum is no distance this run can store:
// float +inf/NaN (never an improvement) or an integer sum that reaches the 32-bit infinity
// value or wraps (the host re-runs with 64-bit distances).  64-bit sums cannot wrap: a distance
// is at most (n-1)(2^32-1) < 2^64 - 2^32.
template <bool kF, typename DistT>
__device__ __forceinline__ DistT relax_narrow(DistT d, unsigned w, bool& bad) {
    if constexpr (kF) {
        const unsigned s = __float_as_uint(__fadd_rn(__uint_as_float((unsigned)d), __uint_as_float(w)));
        bad = s >= 0x7F800000u;
        return (DistT)s;
    } else if constexpr (sizeof(DistT) == 4) {
        const unsigned s = (unsigned)d + w;
        bad = s < w || s == 0xFFFFFFFFu;
        return s;
    } else {
        const unsigned long long s = (unsigned long long)d + w;
        bad = s == ~0ull;
        return s;
    }
}
template <typename DistT>
struct alignas(16) ItemInfo {
    unsigned long long eadj;  // row begin - the item's first arc index in the batch
    DistT d;                  // the item's distance
};

template <bool kF>
__device__ __forceinline__ bool sum_unusable(unsigned long long nd, unsigned long long inf) {
    if constexpr (kF) return nd >= 0x7F800000ull;
    else return nd >= inf;
}
template <bool kF>
__device__ __forceinline__ unsigned bucket_of(unsigned long long nd, unsigned k, unsigned long long h, unsigned nb) {
    if constexpr (kF) {
        const float jf = __uint_as_float((unsigned)nd) * ldexpf(1.0f, kFloatBias - (int)k);  // exact scaling
        const unsigned long long j = jf >= 4.0e18f ? (1ull << 62) : (unsigned long long)jf;
        if (j <= h) return 0u;
        const unsigned long long o = j - h;
        return o >= (unsigned long long)(nb - 1) ? nb - 1 : (unsigned)o;
    } else {
        return adds_bucket_offset(nd, k, h, nb);
    }
}

// --------------------------------------------------------------- 16-bit filter (D11)
// filt[v] = ceil(x / 2^s) for some value x that dist[v] held at some time (so, since
// dist only decreases, filt[v] << s >= dist[v] forever), 0xFFFF = no bound.  The
// relaxation filter reads this 2-byte array (half the L2 footprint of dist) instead
// of dist: nd >= filt[v] << s  =>  nd >= dist[v]  =>  the arc cannot improve.  Any
// racing plain store keeps the invariant, because every value ever written is a
// bound of the (monotone) distance.
__device__ __forceinline__ unsigned long long filt_bound(unsigned short f, unsigned s) {
    return f == 0xFFFFu ? ~0ull : ((unsigned long long)f << s);
}
__device__ __forceinline__ unsigned short filt_enc(unsigned long long x, unsigned s) {
    const unsigned long long q = (x + ((1ull << s) - 1)) >> s;
    return q >= 0xFFFFull ? (unsigned short)0xFFFFu : (unsigned short)q;
}

// --------------------------------------------------------------- claim (A4)
// Warp-cooperative: status + head (lane 0), then the A active buckets' avail
// gates (idle CTAs poll here, so every extra line read lands on a hot L2 slice);
// the highest-priority bucket with published items is claimed: avail -=
// want, give back the excess, claim += got.  Returns got (0 = none); every output
// is warp-uniform: the claim (slot, ring index), the head snapshot and the status.
//
// Hub-split chunks come first (lane 31 polls their gate in the same round trip):
// they are the unfinished rest of an already-claimed item, usually of the head
// bucket, which cannot complete before they do.  A chunk claim returns 1 with
// o_task set and o_idx = the chunk's queue index.
template <typename DistT, int BT, bool kAllGates>
__device__ unsigned claim_batch(const Params<DistT>& p, int lane, unsigned& o_slot, unsigned long long& o_idx,
                                Head& o_head, unsigned& o_status, bool& o_task) {
    o_task = false;
    const unsigned nbm = p.nb - 1;
    unsigned st = 0;
    Head hd{0ull, 0ull};
    // throughput build (kAllGates): one round trip for status + head (lane 0) and every ring
    // slot's avail gate (lane l reads slot l), the active window's gates picked once the head
    // slot is known (RMAT/ER -1 %); latency build: the active gates after the head (its many
    // idle pollers reading 32 hot lines each slowed ROAD 31.2 -> 34.1 ms, sweeps r02 §10)
    long long avs = 0, tv = 0;
    if (lane == 0) {
        st = ld_relaxed_u32(&p.ctl->status);
        hd = ld_head(&p.ctl->head);
    }
    if (kAllGates && lane < (int)p.nb) avs = (long long)ld_relaxed_u64(&p.bk[lane].avail.v);
    if (p.split_deg && lane == 31) tv = (long long)ld_relaxed_u64(&p.bk[kSplitQ].avail.v);
    st = __shfl_sync(FULL, st, 0);
    hd.h = __shfl_sync(FULL, hd.h, 0);
    hd.meta = __shfl_sync(FULL, hd.meta, 0);
    o_status = st;
    o_head = hd;
    if (st) return 0;
    const unsigned hs = meta_hs(hd.meta), A = meta_A(hd.meta);
    long long av;
    if constexpr (kAllGates) {
        av = __shfl_sync(FULL, avs, (int)((hs + (unsigned)lane) & nbm));
        if (lane >= (int)A) av = 0;
    } else {
        av = lane < (int)A ? (long long)ld_relaxed_u64(&p.bk[(hs + lane) & nbm].avail.v) : 0;
    }
    if (__shfl_sync(FULL, tv, 31) > 0) {
        unsigned got = 0;
        unsigned long long ix = 0;
        if (lane == 31) {
            unsigned long long* avp = &p.bk[kSplitQ].avail.v;
            const long long old = (long long)atomicAdd(avp, (unsigned long long)(-1ll));
            if (old > 0) {
                SSSP_FUZZ_AT(FZ_CLAIM);
                ix = atomicAdd(&p.bk[kSplitQ].claim.v, 1ull);
                got = 1;
            } else {
                atomicAdd(avp, 1ull);
            }
        }
        if (__shfl_sync(FULL, got, 31)) {
            o_idx = __shfl_sync(FULL, ix, 31);
            o_slot = 0;
            o_task = true;
            return 1;
        }
    }
    unsigned mask = __ballot_sync(FULL, av > 0);
    while (mask) {
        const int f = __ffs(mask) - 1;
        unsigned g32 = 0, sl32 = 0;
        unsigned long long ix = 0;
        if (lane == f) {
            const unsigned sl = (hs + f) & nbm;
            long long want = av >> p.share_shift;
            if (want < (long long)p.batch_min) want = p.batch_min;
            if (want > BT) want = BT;
            unsigned long long* avp = &p.bk[sl].avail.v;
            const long long old = (long long)atomicAdd(avp, (unsigned long long)(-want));
            const long long g = old <= 0 ? 0 : (old < want ? old : want);
            if (g < want) atomicAdd(avp, (unsigned long long)(want - g));
            if (g > 0) {
                SSSP_FUZZ_AT(FZ_CLAIM);
                ix = atomicAdd(&p.bk[sl].claim.v, (unsigned long long)g);
            }
            g32 = (unsigned)g;
            sl32 = sl;
        }
        g32 = __shfl_sync(FULL, g32, f);
        if (g32) {
            o_idx = __shfl_sync(FULL, ix, f);
            o_slot = __shfl_sync(FULL, sl32, f);
            return g32;
        }
        mask &= mask - 1;
    }
    return 0;
}

// --------------------------------------------------------------- bucket storage
// Where item idx of ring slot sl lives.  Flat (default): slot sl's own array of cap items,
// never lapped within a run (D13).  Chunked: through the slot's chunk table; the chunk is
// published by its reserver before any of its items is stored or claimed, so a wait here is
// only for that publication to become visible.  nullptr = the run was aborted while waiting.
template <typename DistT>
__device__ __forceinline__ char* item_ptr(const Params<DistT>& p, unsigned sl, unsigned long long idx, bool chk) {
    constexpr int kB = ItemT<DistT>::kBytes;
    if (!chk) return p.ring + ((size_t)sl * p.cap + (idx & (p.cap - 1))) * kB;
    const unsigned* e = p.ctab + (size_t)sl * (p.tab_mask + 1) + ((idx >> kChunkShift) & p.tab_mask);
    unsigned id1, spins = 0;
    while ((id1 = ld_acquire_u32(e)) == 0u)
        if ((++spins & 1023) == 0 && ld_relaxed_u32(&p.ctl->status)) return nullptr;
    return p.ring + (((size_t)(id1 - 1) << kChunkShift) + (idx & (kChunkItems - 1))) * kB;
}
// A reserve of [b, b + c) overflows the flat array (no laps, D13); chunked storage overflows
// only when the pool is exhausted (chunk_alloc).
template <typename DistT>
__device__ __forceinline__ bool flat_overflow(const Params<DistT>& p, unsigned long long b, unsigned long long c, bool chk) {
    return !chk && b + c > p.cap;
}
template <typename DistT>
__device__ unsigned chunk_alloc(const Params<DistT>& p) {
    const unsigned long long f = atomicAdd(&p.pool->fresh.v, 1ull);
    if (f < p.pool_chunks) return (unsigned)f;
    const long long old = (long long)atomicAdd(&p.pool->favail.v, (unsigned long long)(-1ll));
    if (old <= 0) {
        atomicAdd(&p.pool->favail.v, 1ull);
        atomicOr(&p.ctl->status, kStRingOverflow);  // pool exhausted: the host doubles it and re-runs
        return 0xFFFFFFFFu;
    }
    const unsigned long long c = atomicAdd(&p.pool->fclaim.v, 1ull);
    unsigned* e = p.free_ring + (c & (p.pool_chunks - 1));
    unsigned id1, spins = 0;
    while ((id1 = ld_acquire_u32(e)) == 0u)
        if ((++spins & 1023) == 0 && ld_relaxed_u32(&p.ctl->status)) return 0xFFFFFFFFu;
    st_relaxed_u32(e, 0u);
    return id1 - 1;
}
// After a reserve of [b, b + c) in slot sl: take every chunk whose first index is in the range
// (the range that reserved a chunk's first index is its only taker).
template <typename DistT>
__device__ void chunks_for_range(const Params<DistT>& p, unsigned sl, unsigned long long b, unsigned long long c,
                                 bool chk) {
    if (!chk || c == 0) return;
    for (unsigned long long ci = (b + kChunkItems - 1) >> kChunkShift; (ci << kChunkShift) < b + c; ++ci) {
        const unsigned id = chunk_alloc(p);
        if (id == 0xFFFFFFFFu) return;
        unsigned* e = p.ctab + (size_t)sl * (p.tab_mask + 1) + (ci & p.tab_mask);
        // the table entry of chunk ci - T must be free by now (T >= pool chunks); if a lagging
        // reader still held it, abort the run rather than alias two chunks
        if (atomicCAS(e, 0u, id + 1) != 0u) atomicOr(&p.ctl->status, kStRingOverflow);
    }
}
// Chunk id (+1) of item idx of slot sl, waiting for its publication (0 = aborted run).
template <typename DistT>
__device__ __forceinline__ unsigned chunk_of(const Params<DistT>& p, unsigned sl, unsigned long long idx) {
    const unsigned* e = p.ctab + (size_t)sl * (p.tab_mask + 1) + ((idx >> kChunkShift) & p.tab_mask);
    unsigned id1, spins = 0;
    while ((id1 = ld_acquire_u32(e)) == 0u)
        if ((++spins & 1023) == 0 && ld_relaxed_u32(&p.ctl->status)) return 0u;
    return id1;
}
template <typename DistT>
__device__ __forceinline__ char* chunk_item(const Params<DistT>& p, unsigned id1, unsigned long long idx) {
    return p.ring + (((size_t)(id1 - 1) << kChunkShift) + (idx & (kChunkItems - 1))) * ItemT<DistT>::kBytes;
}

// Thread 0, after the CTA barrier that follows a pop of [idx0, idx0 + got) in slot sl (every
// item read and cleared): count the reads per chunk; the reader that completes a chunk frees it.
template <typename DistT>
__device__ void chunks_consumed(const Params<DistT>& p, unsigned sl, unsigned long long idx0, unsigned got) {
    const unsigned long long end = idx0 + got;
    for (unsigned long long i = idx0; i < end;) {
        const unsigned long long cend = ((i >> kChunkShift) + 1) << kChunkShift;
        const unsigned cnt = (unsigned)((cend < end ? cend : end) - i);
        unsigned* e = p.ctab + (size_t)sl * (p.tab_mask + 1) + ((i >> kChunkShift) & p.tab_mask);
        const unsigned id1 = ld_relaxed_u32(e);  // still ours: not all of its items are counted yet
        __threadfence();                         // the CTA's clears (barrier-ordered) before the count
        if (atomicAdd(p.chunk_used + (id1 - 1), cnt) + cnt == kChunkItems) {
            p.chunk_used[id1 - 1] = 0;
            st_relaxed_u32(e, 0u);
            __threadfence();
            const unsigned long long r = atomicAdd(&p.pool->freserve.v, 1ull);
            st_release_u32(p.free_ring + (r & (p.pool_chunks - 1)), id1);
            atomicAdd(&p.pool->favail.v, 1ull);
        }
        i += cnt;
    }
}

// --------------------------------------------------------------- hub split (A5)
// Publish arcs [S, deg) of vertex v (expanded at distance d, row begins at b) as
// chunks of S arcs; the caller processes the first S itself.  The chunks are
// charged to the item's ring slot BEFORE they become claimable, so the bucket
// stays incomplete (the head cannot pass it) until every chunk is done.
template <typename DistT>
__device__ unsigned spawn_chunks(const Params<DistT>& p, unsigned v, unsigned long long d, unsigned long long b,
                                 unsigned deg, unsigned slot) {
    const unsigned S = p.split_deg;
    const unsigned extra = (deg - 1) / S;
    atomicAdd(&p.bk[slot].local.v, (unsigned long long)extra);
    const unsigned long long t0 = atomicAdd(&p.bk[kSplitQ].reserve.v, (unsigned long long)extra);
    SSSP_FUZZ_AT(FZ_CHUNK);
    if (t0 + extra > p.tcap && t0 + extra - p.tcap > ld_relaxed_u64(&p.bk[kSplitQ].claim.v)) {
        atomicOr(&p.ctl->status, kStRingOverflow);  // would lap an unclaimed chunk: regrow and re-run
        return S;
    }
    for (unsigned c = 1; c <= extra; ++c) {
        const unsigned long long idx = t0 + c - 1;
        SplitTask* tp = p.tasks + (idx & (p.tcap - 1));
        // take the slot (free -> busy); it is still occupied while the previous lap's
        // chunk has not been read
        unsigned spins = 0;
        while (atomicCAS(&tp->len, 0u, kLenBusy) != 0u)
            if ((++spins & 255) == 0 && ld_relaxed_u32(&p.ctl->status)) return S;
        tp->beg = b + (unsigned long long)c * S;
        tp->d = d;
        tp->v = v;
        tp->slot = slot;
    }
    __threadfence();  // payloads before their len markers
    SSSP_FUZZ_AT(FZ_CHUNK);
    for (unsigned c = 1; c <= extra; ++c) {
        const unsigned rest = deg - c * S;
        st_relaxed_u32(&p.tasks[(t0 + c - 1) & (p.tcap - 1)].len, rest < S ? rest : S);
    }
    atomicAdd(&p.bk[kSplitQ].avail.v, (unsigned long long)extra);
    return S;
}

// Take a published chunk (CAS len -> reading, acquire); returns its length, or 0
// if the run was aborted while waiting.  The caller reads the payload and frees
// the slot with a release store of 0 (common.cuh, kLenReading).
template <typename DistT>
__device__ __forceinline__ unsigned take_chunk(const Params<DistT>& p, SplitTask* tp) {
    unsigned spins = 0;
    for (;;) {
        const unsigned len = ld_relaxed_u32(&tp->len);
        if (len != 0u && len != kLenBusy && len != kLenReading && cas_acquire_u32(&tp->len, len, kLenReading) == len)
            return len;
        if ((++spins & 1023) == 0 && ld_relaxed_u32(&p.ctl->status)) return 0u;
    }
}

// --------------------------------------------------------------- shared memory
constexpr size_t align16(size_t x) { return (x + 15) & ~(size_t)15; }

template <typename DistT, int BT, int EPT>
struct Smem {
    using Raw = typename ItemT<DistT>::Raw;
    // staged ring pushes of one batch (beyond this, warps publish directly)
    // (shared memory is taken from the L1 that holds in-flight misses: keep it small)
    static constexpr int kStage = STAGE_MULT * BT * EPT / 2;
    static constexpr size_t o_arc = 0;                                        // (no arc window)
    static constexpr size_t o_items = 0;                                      // Raw[kStage] staged pushes
    // per expanded item (compacted: items with at least one arc, in scan order)
    static constexpr size_t o_info = o_items + align16((size_t)kStage * sizeof(Raw));  // ItemInfo[BT]
    static constexpr size_t o_ld = o_info + (size_t)BT * 16;                  // DistT[BT] kept children
    static constexpr size_t o_owner = o_ld + align16((size_t)BT * sizeof(DistT));  // (unused)
    static constexpr size_t o_rank = o_owner;                                 // u16[kStage]
    static constexpr size_t o_scan = o_rank + align16((size_t)kStage * 2);    // u32[BT+1] arc offsets, sentinel E
    static constexpr size_t o_lv = o_scan + align16((size_t)(BT + 1) * 4);    // u32[BT] kept children
    static constexpr size_t o_soff = o_lv + align16((size_t)BT * 4);          // u8[kStage]
    // warp-local continuation queues: kWQ {vertex, distance, row begin, degree} per warp
    // (the row is fetched when the child is found, so a hop starts with its arc loads)
    static constexpr int kWQ = 96;
    static constexpr size_t o_wqv = o_soff + align16((size_t)kStage);         // u32[BT/32 * kWQ]
    static constexpr size_t o_wqd = o_wqv + align16((size_t)(BT / 32) * kWQ * 4);  // DistT[BT/32 * kWQ]
    static constexpr size_t o_wqb = o_wqd + align16((size_t)(BT / 32) * kWQ * sizeof(DistT));  // u64[]
    static constexpr size_t o_wqn = o_wqb + (size_t)(BT / 32) * kWQ * 8;      // u32[]
    static constexpr size_t bytes = o_wqn + align16((size_t)(BT / 32) * kWQ * 4);
};

// --------------------------------------------------------------- kernel
// BT threads per CTA, EPT arcs per thread per round, MINB CTAs per SM (register
// budget 65536 / (MINB * BT)), PIPE: the arc loads of a warp's next round are
// issued before the current round's gathers/atomics (software pipeline: one
// fewer dependent L2/HBM trip per round), kF: float32 weights (NEXT-3).
// WLC: the warp-local continuation loop is compiled in (latency-regime graphs); the
// throughput build leaves it out so its register allocation is not shaped by it.
// CA: claim-ahead in the throughput regime -- warp 0 claims the next batch as soon as it
// has streamed its own slice of the current one, so the claim round trips overlap the
// other warps' streaming, the flush and the completion (held for the tail of one batch
// only; claiming at the start of a batch held the claim too long, sweeps §7).
// CHM: bucket storage -- 0 flat no-lap arrays, 1 chunked pool, 2 chosen at run time (p.chunked);
// the product's default builds are compiled for 0 and 1 so the flat path carries no chunk code.
template <typename DistT, int BT, int EPT, int MINB, bool PIPE, bool kF, bool WLC = true, bool CA = false, int CHM = 2>
__global__ void __launch_bounds__(BT, MINB) adds_persistent_kernel(const Params<DistT> p) {
    // items per thread: one (batches of two items per thread, to pay the per-batch round
    // trips half as often, measured slower -- ER 13.1 vs 11.4 ms -- from register spills)
    using IT = ItemT<DistT>;
    using Raw = typename IT::Raw;
    using L = Smem<DistT, BT, EPT>;
    constexpr int kStage = L::kStage;
    constexpr int kWarps = BT / 32;
    constexpr unsigned long long kInf = (unsigned long long)DistInf<DistT>::value;

    extern __shared__ __align__(16) unsigned char smem[];
    Raw* s_items = (Raw*)(smem + L::o_items);
    // per expanded item, one 16-byte shared load per arc: {row begin - arc offset, distance}
    ItemInfo<DistT>* s_info = (ItemInfo<DistT>*)(smem + L::o_info);
    DistT* s_ld = (DistT*)(smem + L::o_ld);
    unsigned short* s_rank = (unsigned short*)(smem + L::o_rank);
    unsigned* s_scan = (unsigned*)(smem + L::o_scan);
    unsigned* s_lv = (unsigned*)(smem + L::o_lv);
    unsigned char* s_soff = (unsigned char*)(smem + L::o_soff);
    constexpr unsigned kWQ = (unsigned)L::kWQ;
    unsigned* s_wqv = (unsigned*)(smem + L::o_wqv);
    DistT* s_wqd = (DistT*)(smem + L::o_wqd);
    unsigned long long* s_wqb = (unsigned long long*)(smem + L::o_wqb);
    unsigned* s_wqn = (unsigned*)(smem + L::o_wqn);
    __shared__ unsigned s_wst[5];  // warp-local continuation: expanded, first, edges, stale, kept

    // staging: warp w owns s_items[w * kSeg, (w + 1) * kSeg) and its fill is a register;
    // s_wcnt[w][o] = items warp w staged for bucket o (its ranks), turned into the warp's
    // offset inside the CTA's reservation of bucket o at flush time
    constexpr unsigned kSeg = (unsigned)kStage / kWarps;
    static_assert(32 % kWarps == 0, "warps per CTA must divide 32");
    __shared__ unsigned s_wcnt[kWarps][kMaxBuckets];
    __shared__ unsigned s_cnt[kMaxBuckets];
    __shared__ unsigned long long s_base[kMaxBuckets];
    // chunks one CTA reservation (<= kStage items) can span
    constexpr unsigned kFlushChunks = ((unsigned)kStage + kChunkItems - 1) / kChunkItems + 1;
    __shared__ unsigned s_cid[kMaxBuckets][kFlushChunks];                  // chunked storage: their ids
    __shared__ unsigned s_wsum[kWarps], s_wnz[kWarps];
    __shared__ unsigned s_total, s_got, s_slot, s_lnext, s_direct, s_task, s_tslot;
    __shared__ unsigned s_fin;  // warps done streaming this batch (first-finisher claim-ahead)
    __shared__ volatile unsigned s_ahead;  // (own load: not merged with the claim fields)
    __shared__ int s_cmd[2];  // by loop parity: an idle CTA loops back to the claim with no
                              // second barrier, so the next claim must not overwrite the
                              // value a slow warp is still to read (compute-sanitizer racecheck)
    unsigned par = 0;
    __shared__ unsigned long long s_idx;
    __shared__ Head s_head;
    __shared__ unsigned long long s_prof[kProfCounters];

    // throughput build with 32-bit row records (m < 2^32): 8-byte pops of {begin, degree},
    // 8-byte per-item records {row begin - arc offset, distance}, 32-bit bucket arithmetic
    constexpr bool kTP = !WLC && CA && !kF && sizeof(DistT) == 4;
    uint2* s_info2 = (uint2*)(smem + L::o_info);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const unsigned lt_mask = lanemask_lt();
    const unsigned le_mask = lt_mask | (1u << lane);
    const bool chk = CHM == 2 ? p.chunked != 0 : CHM == 1;  // chunked bucket storage
    const unsigned nbm = p.nb - 1;
    const unsigned local_max = p.local_max < (unsigned)BT ? p.local_max : (unsigned)BT;
    unsigned long long c_vert = 0, c_edges = 0, c_push = 0, c_stale = 0, c_local = 0;  // thread 0
    unsigned backoff = 0;
    const bool track_busy = p.dynamic && p.adapt_active;
    bool busy_cta = false;  // warp 0 lane 0: this CTA is counted in g_busy
    unsigned have_local = 0;  // uniform: items of the next batch already in s_lv/s_ld
    unsigned kslot = 0;       // their ring slot (the batch's own)
    __shared__ unsigned s_nf;  // first expansions of this batch (controller), summed per warp

    if (tid < (int)kMaxBuckets) s_cnt[tid] = 0;
    for (int i = tid; i < kWarps * (int)kMaxBuckets; i += BT) (&s_wcnt[0][0])[i] = 0;
    if (tid < (int)kProfCounters) s_prof[tid] = 0;
    if (tid < 5) s_wst[tid] = 0;
    if (tid == 0) {
        s_total = 0;
        s_lnext = 0;
        s_direct = 0;
        s_ahead = 0;
        s_fin = 0;
        s_nf = 0;
    }
    const bool prof = p.prof != 0 && tid == 0;
    const unsigned long long pol_stream = policy_evict_first();  // arcs, row offsets
    const unsigned long long pol_keep = policy_evict_last(p.keep_frac);  // dist
    const long long t_begin = clock64();
    long long t0 = t_begin, tq = 0, tw = 0;
    __syncthreads();

    for (;;) {
        unsigned got, slot;
        bool from_ring, is_task = false;
        bool ahead = false;  // this batch is the one claimed ahead
        if (prof) t0 = clock64();
        if (have_local) {
            got = have_local;
            slot = kslot;
            from_ring = false;
        } else if (CA && s_ahead) {  // claimed ahead during a previous batch
            ahead = true;
            got = s_got;
            slot = s_slot;
            from_ring = true;
            is_task = s_task != 0;
        } else {
            // -------------------------------------------------------- claim
            if (warp == 0) {
                int cmd = CMD_IDLE;
                unsigned sl = 0, st = 0;
                unsigned long long idx = 0;
                Head hd;
                bool tk;
                const unsigned g = claim_batch<DistT, BT, !WLC>(p, lane, sl, idx, hd, st, tk);
                if (st) {
                    cmd = CMD_EXIT;
                } else if (g) {
                    cmd = CMD_WORK;
                    if (lane == 0) {
                        if (track_busy && !busy_cta) {  // idle -> holding work (utilisation)
                            red_add_u64(&p.ctl->g_busy, 1ull);
                            busy_cta = true;
                        }
                        s_got = g;
                        s_slot = sl;
                        s_idx = idx;
                        s_head = hd;
                        s_task = tk ? 1u : 0u;
                        backoff = 0;
                    }
                } else {
                    if (try_advance<DistT>(p, hd, lane)) {
                        cmd = CMD_EXIT;
                    } else if (lane == 0) {
                        if (track_busy && busy_cta) {  // found nothing to claim: idle
                            red_add_u64(&p.ctl->g_busy, ~0ull);
                            busy_cta = false;
                        }
                        if (globaltimer() - p.ctl->t_start > p.timeout_ns) atomicOr(&p.ctl->status, kStTimeout);
                        backoff = backoff ? (backoff * 2 < p.max_backoff_ns ? backoff * 2 : p.max_backoff_ns) : 32;
                        __nanosleep(backoff);
                    }
                }
                if (lane == 0) s_cmd[par] = cmd;
            }
            __syncthreads();
            const int cmd = s_cmd[par];
            par ^= 1u;
            if (prof) {
                const long long t1 = clock64();
                s_prof[cmd == CMD_WORK ? PR_CLAIM : PR_IDLE] += t1 - t0;
                if (cmd == CMD_IDLE) s_prof[PR_N_IDLE] += 1;
                t0 = t1;
            }
            if (cmd == CMD_EXIT) break;
            if (cmd == CMD_IDLE) continue;
            got = s_got;
            slot = s_slot;
            from_ring = true;
            is_task = s_task != 0;
        }

        // CTA-local continuation only in the latency regime (small batches = scarce
        // work): with plentiful work it starves the other CTAs of head-bucket items
        // (measured: RMAT 2x slower with a full-CTA cap)
        const unsigned lcap = got * 2 <= (unsigned)BT ? local_max : 0u;
        // warp-local continuation (same regime): a warp runs its own head-bucket
        // children hop after hop with no CTA barrier (D9)
        const bool wlc = WLC && lcap != 0 && p.warp_local != 0;

        // ------------------------------------------------------------ pop + stale check
        const Head hd = s_head;
        const unsigned hs = meta_hs(hd.meta), k = meta_k(hd.meta);
        const unsigned h32 = hd.h > 0xFFFFFFFFull ? 0xFFFFFFFFu : (unsigned)hd.h;  // (32-bit distances: j <= h32 iff j <= h)
        unsigned deg = 0;               // arcs this thread's item contributes to the batch
        bool live = false;              // the item is expanded (not stale)
        unsigned long long my_b = 0;    // its row begin
        unsigned long long my_d = 0;    // its distance
        unsigned fword = 0, fbit = 0;   // expansion-bitmap word before our atomicOr (consumed at batch end)
        if (is_task) {
            // a hub-split chunk: one vertex, len arcs, charged to the slot it carries
            if (tid == 0) {
                SplitTask* tp = p.tasks + (s_idx & (p.tcap - 1));
                s_tslot = 0;  // (not s_slot: other threads may still be reading it)
                const unsigned len = take_chunk(p, tp);
                if (len) {
                    const unsigned long long b = __ldcg(&tp->beg), d = __ldcg(&tp->d);
                    const unsigned v = __ldcg(&tp->v);
                    s_tslot = __ldcg(&tp->slot);
                    st_release_u32(&tp->len, 0u);  // free the slot after the read
                    const unsigned long long cur = (unsigned long long)ld_keep(p.dist + v, pol_keep);
                    if (cur >= d) {  // stale chunks (v improved since) are dropped
                        deg = len;
                        my_b = b;
                        my_d = d;
                        live = true;
                    }
                }
            }
        } else {
            if (tid < (int)got) {
                uint32_t v;
                unsigned long long d;
                bool loaded = true;
                if (from_ring) {
                    char* sp = item_ptr(p, slot, s_idx + tid, chk);
                    unsigned spins = 0;
                    SSSP_FUZZ_AT(FZ_POP);
                    loaded = false;
                    while (sp && !(loaded = IT::load(sp, v, d))) {  // reserved, store not landed yet
                        if ((++spins & 1023) == 0 && ld_relaxed_u32(&p.ctl->status)) break;  // aborted run
                    }
                    if (loaded) IT::clear(sp);  // the slot's one reader this run (D13)
                } else {
                    v = s_lv[tid];
                    d = (unsigned long long)s_ld[tid];
                }
                if (loaded) {
                    // the stale check and the row loads are independent: one round trip
                    const unsigned long long cur = (unsigned long long)ld_keep(p.dist + v, pol_keep);
                    unsigned long long b, e;
                    if constexpr (kTP) {
                        const uint2 r = ld_stream_u2(p.rows + v, pol_stream);
                        b = r.x;
                        e = (unsigned long long)r.x + r.y;
                    } else {
                        b = ld_stream_u64(p.off + v, pol_stream);
                        e = ld_stream_u64(p.off + v + 1, pol_stream);
                    }
                    if (cur >= d) {  // not stale: d is still v's distance ("refined")
                        deg = (unsigned)(e - b);
                        my_b = b;
                        my_d = d;
                        live = true;
                        if (p.dynamic) {  // work-waste signal: is this v's first expansion?
                            fbit = 1u << (v & 31);
                            fword = atomicOr(p.expanded + (v >> 5), fbit);  // result not waited for until the batch ends
                        }
                        if (p.split_deg && deg > p.split_deg) deg = spawn_chunks(p, v, d, b, deg, slot);
                    }
                }
            }
        }
        if (prof) {
            const long long t1 = clock64();
            s_prof[PR_POP] += t1 - t0;
            s_prof[from_ring ? PR_N_RING : PR_N_LOCAL] += 1;
            t0 = t1;
        }
        // exclusive scan of degrees over the CTA, and the items with arcs compacted in
        // scan order (rank r): s_scan[r] = first arc of item r in the batch's arc space,
        // strictly increasing, with the sentinel s_scan[NZ] = E -- the owner search of the
        // streaming loop relies on distinct starts (one bit per item start, below)
        unsigned x = deg;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned y = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += y;
        }
        const unsigned nzm = __ballot_sync(FULL, deg > 0);
        if (lane == 31) {
            s_wsum[warp] = x;
            s_wnz[warp] = __popc(nzm);
        }
        const int nlive = __syncthreads_count(live);
        // (every thread read the last batch's s_lnext before this barrier: no barrier ends a batch)
        if (tid == 0) s_lnext = 0;
        // chunked storage: this batch's reads (and clears) are complete; count them per chunk
        if (chk && tid == 0 && from_ring && !is_task) chunks_consumed(p, slot, s_idx, got);
        // every warp combines the kWarps warp totals itself (four warp reductions), so no warp
        // waits on a serial scan by warp 0 and one barrier is saved
        const unsigned ws = lane < kWarps ? s_wsum[lane] : 0u;
        const unsigned wn = lane < kWarps ? s_wnz[lane] : 0u;
        const unsigned E = __reduce_add_sync(FULL, ws), NZ = __reduce_add_sync(FULL, wn);
        const unsigned wpre = __reduce_add_sync(FULL, lane < warp ? ws : 0u);
        const unsigned wnpre = __reduce_add_sync(FULL, lane < warp ? wn : 0u);
        if (tid == 0) s_scan[NZ] = E;  // sentinel
        if (deg > 0) {
            const unsigned r = wnpre + __popc(nzm & lt_mask);
            const unsigned ex = x - deg + wpre;
            s_scan[r] = ex;
            if constexpr (kTP) s_info2[r] = make_uint2((unsigned)my_b - ex, (unsigned)my_d);  // (mod 2^32)
            else s_info[r] = ItemInfo<DistT>{my_b - ex, (DistT)my_d};  // arc e of the batch is adj[eadj + e]
        }
        if (is_task) slot = s_tslot;
        const int nexp = is_task ? 0 : nlive;  // a chunk is not a vertex expansion
        if (tid == 0) {
            c_vert += nexp;
            if (!is_task) c_stale += got - nlive;
            c_edges += E;
        }
        if (prof) {
            const long long t1 = clock64();
            s_prof[PR_SCAN] += t1 - t0;
            t0 = t1;
            tq = 0;
            tw = 0;
        }

        __syncthreads();  // publishes s_scan / s_info
        if (CA && ahead && tid == 0) s_ahead = 0;  // every thread has read it (loop top)
        unsigned wfill = 0;  // warp-uniform: items staged in this warp's segment
        // ---------------------------------------------------- stream the batch's arcs
        // Warp w owns a contiguous slice of the batch's arc space and streams through
        // it with no CTA barrier (warps drift and keep the L1TEX queue busy); lanes
        // take consecutive arcs (coalesced along rows), EPT in flight per lane; the
        // owner of an arc is found by binary search over the CTA scan in shared memory.
        // Tiny batches (latency regime, road-like graphs) skip the L2 filter load.
        {
            const bool tiny = E <= (unsigned)BT;
            // static slices (dynamic 32*EPT-arc chunks from a shared counter measured
            // neutral on RMAT/ER, profiles/r01_sweeps.md §14)
            constexpr unsigned kChunk = 32u * EPT;
            const unsigned per = (E + kWarps - 1) / kWarps;
            const unsigned slice = (per + 31) / 32 * 32;  // small batches spread over many warps
            const unsigned wb = warp * slice;
            const unsigned we = (wb + slice) < E ? (wb + slice) : E;
            // Owner of each arc = the largest r with s_scan[r] <= e.  The warp walks its
            // slice in windows of 32 consecutive arcs (one per lane) and carries `cur`, the
            // owner of the window's first arc: lane l reads the start of item cur+1+l, the
            // starts inside the window become one bit each (they are distinct), and an arc's
            // owner is cur + the number of starts at or before it -- one shared load, one
            // warp OR-reduction and a popcount per arc instead of a binary search
            // (log2(BT) dependent shared loads per arc).  One binary search per slice.
            unsigned cur = 0;
            if (wb < we) {
                unsigned lo = 0, hi = NZ - 1;
                while (lo < hi) {
                    const unsigned mid = (lo + hi + 1) >> 1;
                    if (s_scan[mid] <= wb) lo = mid;
                    else hi = mid - 1;
                }
                cur = lo;
            }
            auto fetch = [&](unsigned base, DistT (&dv)[EPT], uint2 (&a)[EPT]) {
                unsigned own[EPT];
#pragma unroll
                for (int j = 0; j < EPT; ++j) {
                    const unsigned w0 = base + j * 32;
                    const unsigned ix = cur + 1 + lane;
                    const unsigned rel = s_scan[ix < NZ ? ix : NZ] - w0;  // >= 1 while w0 < E
                    const unsigned bits = __reduce_or_sync(FULL, rel < 32u ? 1u << rel : 0u);
                    own[j] = cur + __popc(bits & le_mask);
                    cur += __popc(__ballot_sync(FULL, rel <= 32u));  // owner of the next window's first arc
                }
#pragma unroll
                for (int j = 0; j < EPT; ++j) {  // EPT independent arc loads in flight
                    const unsigned e = base + j * 32 + lane;
                    if constexpr (kTP) {
                        const uint2 ii = s_info2[min(own[j], NZ - 1u)];
                        a[j] = ld_stream_u2_if(e < we, p.adj + (ii.x + e), pol_stream);
                        dv[j] = (DistT)ii.y;
                    } else {
                        a[j] = make_uint2(0u, 0u);
                        dv[j] = (DistT)0;
                        if (e < we) {
                            const ItemInfo<DistT> ii = s_info[own[j]];
                            a[j] = ld_stream_u2(p.adj + (ii.eadj + e), pol_stream);
                            dv[j] = ii.d;
                        }
                    }
                }
            };
            // head-bucket children stay on chip: first in this warp's own queue (warp-local
            // continuation), then in the CTA's next batch (warp-aggregated slot grabs)
            unsigned wq_n = 0;  // warp-uniform fill of this warp's queue
            unsigned wq_h = 0;  // logical index of its oldest entry (entries: [wq_h, wq_h + wq_n) mod kWQ)
            const unsigned wq0 = (unsigned)warp * kWQ;
            // oldest first: an item that waited longest is the one most likely to hold the
            // bucket open (FIFO vs LIFO on ROAD static 2^12: 34.4 vs 35.3 ms, sweeps §22);
            // past the queue depth children go to the CTA's next batch (shared by all warps)
            // or the ring (other CTAs)
            constexpr unsigned wqcap = kWQ;
            // rb/rn: the child's row (begin, degree) when already fetched (has_row), else it
            // is loaded here
            auto keep = [&](const bool want, const unsigned v, const unsigned long long ndv, const bool has_row,
                            unsigned long long rb, unsigned rn) -> bool {
                bool kept = false;
                if (wlc) {
                    const unsigned wm = __ballot_sync(FULL, want);
                    if (wm) {
                        const unsigned pos = wq_n + __popc(wm & lt_mask);
                        const unsigned ph = wq0 + (wq_h + pos) % kWQ;
                        if (want && pos < wqcap) {
                            if (!has_row) {
                                rb = ld_stream_u64(p.off + v, pol_stream);
                                rn = (unsigned)(ld_stream_u64(p.off + v + 1, pol_stream) - rb);
                            }
                            s_wqv[ph] = v;
                            s_wqd[ph] = (DistT)ndv;
                            s_wqb[ph] = rb;
                            s_wqn[ph] = rn;
                            kept = true;
                        }
                        const unsigned nn = wq_n + __popc(wm);
                        if (lane == 0) atomicAdd(&s_wst[4], (nn < wqcap ? nn : wqcap) - wq_n);
                        wq_n = nn < wqcap ? nn : wqcap;
                    }
                }
                if (lcap) {
                    const bool w2 = want && !kept;
                    const unsigned lm = __ballot_sync(FULL, w2);
                    if (lm) {
                        const int leader = __ffs(lm) - 1;
                        unsigned pos = 0;
                        if (lane == leader) pos = atomicAdd(&s_lnext, (unsigned)__popc(lm));
                        pos = __shfl_sync(FULL, pos, leader) + __popc(lm & lt_mask);
                        if (w2 && pos < lcap) {
                            s_lv[pos] = v;
                            s_ld[pos] = (DistT)ndv;
                            kept = true;
                        }
                    }
                }
                return kept;
            };
            // A full segment is published by its warp alone (warp_flush): one reserve and one
            // avail atomic per bucket present, coalesced stores -- 32x fewer round trips than
            // publishing each push directly.  The children are counted (reserve) before this
            // batch's completion, as at the CTA flush.
            // Rank the warp's staged items within their buckets (s_rank) and count them per
            // bucket (s_wcnt[warp]): deferred from the push sites to here, where a warp-wide
            // match_any covers 32 staged items instead of the one or two pushes of a site.
            auto rank_segment = [&]() {
                __syncwarp();  // staged entries written by other lanes (emit) are visible
                for (unsigned i0 = 0; i0 < wfill; i0 += 32) {
                    const unsigned i = i0 + (unsigned)lane;
                    const unsigned my = (unsigned)warp * kSeg + i;
                    const bool valid = i < wfill;
                    const unsigned o = valid ? s_soff[my] : 0xFFu;
                    const unsigned peers = __match_any_sync(FULL, o);
                    const int pl = __ffs(peers) - 1;
                    unsigned r0 = 0;
                    if (valid && lane == pl) {  // one lane per distinct bucket
                        r0 = s_wcnt[warp][o];
                        s_wcnt[warp][o] = r0 + (unsigned)__popc(peers);
                    }
                    r0 = __shfl_sync(FULL, r0, pl) + __popc(peers & lt_mask);
                    if (valid) s_rank[my] = (unsigned short)r0;
                    __syncwarp();
                }
            };
            auto warp_flush = [&]() {
                rank_segment();
                const unsigned c = lane < (int)p.nb ? s_wcnt[warp][lane] : 0u;
                const unsigned sl = (hs + (unsigned)lane) & nbm;
                unsigned long long b = 0;
                if (c) {
                    b = atomicAdd(&p.bk[sl].reserve.v, (unsigned long long)c);
                    SSSP_FUZZ_AT(FZ_RESERVE);
                    if (flat_overflow(p, b, c, chk)) atomicOr(&p.ctl->status, kStRingOverflow);  // no laps (D13)
                    chunks_for_range(p, sl, b, c, chk);
                    if (p.dynamic && lane == (int)nbm) atomicAdd(&p.ctl->g_clip, (unsigned long long)c);
                }
                // chunked storage: a segment's range spans at most two chunks (kSeg <= kChunkItems)
                unsigned cid0 = 0, cid1 = 0;
                if (chk && c) {
                    cid0 = chunk_of(p, sl, b);
                    if (((b + c - 1) >> kChunkShift) != (b >> kChunkShift)) cid1 = chunk_of(p, sl, b + c - 1);
                }
                for (unsigned i0 = 0; i0 < wfill; i0 += 32) {
                    const unsigned i = i0 + (unsigned)lane;
                    const unsigned my = (unsigned)warp * kSeg + i;
                    const unsigned o = i < wfill ? s_soff[my] : 0u;
                    const unsigned long long bo = __shfl_sync(FULL, b, (int)o);
                    const unsigned c0 = __shfl_sync(FULL, cid0, (int)o), c1 = __shfl_sync(FULL, cid1, (int)o);
                    if (i < wfill) {
                        const unsigned long long idx = bo + s_rank[my];
                        SSSP_FUZZ_AT(FZ_PUBLISH);
                        // the slot's one writer this run (D13); beyond cap the run is aborted
                        if (chk) {
                            const unsigned id1 = ((idx >> kChunkShift) == (bo >> kChunkShift)) ? c0 : c1;
                            if (id1) IT::store(chunk_item(p, id1, idx), s_items[my]);
                        } else if (idx < p.cap) {
                            IT::store(item_ptr(p, (hs + o) & nbm, idx, chk), s_items[my]);
                        }
                    }
                }
                __syncwarp();
                if (c) atomicAdd(&p.bk[sl].avail.v, (unsigned long long)c);  // publish
                if (lane < (int)p.nb) s_wcnt[warp][lane] = 0;
                if (lane == 0) atomicAdd(&s_direct, wfill);
                wfill = 0;
                __syncwarp();
            };
            // everything else: staged in the warp's own segment for the CTA flush at batch
            // end (no shared atomics: the fill is a warp-uniform register; bucket ranks and
            // counts are computed at flush time)
            auto emit = [&](const bool pg, const unsigned v, const unsigned long long ndv, const unsigned o) {
                const unsigned act = __ballot_sync(FULL, pg);
                if (!act) return;
                const unsigned nact = (unsigned)__popc(act);
                if (wfill + nact > kSeg) {
                    if constexpr (WLC) {
                        // latency build: segments rarely fill; publish just these pushes
                        // (keeps the warp-local hop loop short, ROAD 33.8 vs 32.2 ms with
                        // warp_flush here)
                        if (pg) {
                            const unsigned peers = __match_any_sync(act, o);
                            const int pl = __ffs(peers) - 1;
                            const unsigned sl = (hs + o) & nbm;
                            unsigned long long b0 = 0;
                            if (lane == pl) {
                                const unsigned c = (unsigned)__popc(peers);
                                b0 = atomicAdd(&p.bk[sl].reserve.v, (unsigned long long)c);
                                if (flat_overflow(p, b0, c, chk)) atomicOr(&p.ctl->status, kStRingOverflow);  // no laps (D13)
                                chunks_for_range(p, sl, b0, c, chk);
                                atomicAdd(&s_direct, c);
                                SSSP_FUZZ_AT(FZ_RESERVE);
                            }
                            b0 = __shfl_sync(peers, b0, pl);
                            const unsigned long long idx = b0 + __popc(peers & lt_mask);
                            // the slot's one writer this run (D13); beyond cap the run is aborted
                            if (chk || idx < p.cap) {
                                char* ip = item_ptr(p, sl, idx, chk);
                                if (ip) IT::store(ip, IT::make(v, ndv));
                            }
                            SSSP_FUZZ_AT(FZ_PUBLISH);
                            __syncwarp(peers);
                            if (lane == pl) atomicAdd(&p.bk[sl].avail.v, (unsigned long long)__popc(peers));
                        }
                        return;
                    } else {
                        warp_flush();
                    }
                }
                if (pg) {  // (bucket ranks are assigned at flush time, rank_segment)
                    const unsigned my = (unsigned)warp * kSeg + wfill + __popc(act & lt_mask);
                    s_items[my] = IT::make(v, ndv);
                    s_soff[my] = (unsigned char)o;
                }
                wfill += nact;
            };
            // relax + push of one round whose arcs are loaded
            // Relaxation write (A6).  With a gathered dist value cur (the plain L2 load that
            // filters the atomics) the update is a fire-and-forget RED.min and the arc pushes
            // iff nd < cur: whichever relaxation actually lowers dist[v] to x saw cur > x
            // (dist only decreases), so every value dist[v] takes is pushed by its writer; a
            // relaxation that lost a race to a smaller value pushes an item that is stale at
            // its pop (skipped), or a duplicate of an equal one (expanded twice, same
            // result).  Without the gather (tiny batches) or with the 16-bit filter (cur is
            // only a bound) the returning atomicMin decides.
            const bool fire = !tiny && p.filt == nullptr;
            // (distances in DistT width: d + w is computed in 32 bits for 32-bit distances, an
            // overflow or the infinity value flags a re-run with 64-bit distances)
            auto body = [&](const unsigned base, const DistT (&dv)[EPT], const uint2 (&a)[EPT]) {
                DistT nd[EPT];
                bool live[EPT], bad[EPT];
                bool push[EPT];
                DistT cur[EPT];
#pragma unroll
                for (int j = 0; j < EPT; ++j) {
                    live[j] = base + j * 32 + lane < we;
                    nd[j] = relax_narrow<kF, DistT>(dv[j], a[j].y, bad[j]);
                    bad[j] = bad[j] && live[j];
                    live[j] = live[j] && !bad[j];
                }
#pragma unroll
                for (int j = 0; j < EPT; ++j)  // EPT independent L2 gathers in flight
                    cur[j] = live[j] ? DistInf<DistT>::value : (DistT)0;
                if (!tiny) {
                    if (p.filt == nullptr) {  // (uniform branch: the opt-in filter path stays out of the loop)
#pragma unroll
                        for (int j = 0; j < EPT; ++j)
                            if (live[j]) cur[j] = ld_keep(p.dist + a[j].x, pol_keep);
                    } else {
#pragma unroll
                        for (int j = 0; j < EPT; ++j)
                            if (live[j])
                                cur[j] = (DistT)min(filt_bound(ld_filt(p.filt + a[j].x), p.filt_shift),
                                                    (unsigned long long)DistInf<DistT>::value);
                    }
                }
                DistT old[EPT];
                bool tried[EPT];
#pragma unroll
                for (int j = 0; j < EPT; ++j) {  // all atomics issued before any result is used
                    tried[j] = false;
                    old[j] = (DistT)0;
                    if (bad[j]) {
                        if (!kF) atomicOr(&p.ctl->status, kStDistOverflow);  // 32-bit distances insufficient
                    } else if (live[j]) {
                        if (nd[j] < cur[j]) {
                            if (fire) {
                                // fire-and-forget (D19): push on the gathered value; the RED
                                // needs no round trip
                                red_min_keep(p.dist + a[j].x, nd[j], pol_keep);
                                old[j] = cur[j];
                            } else {
                                old[j] = atomic_min_keep(p.dist + a[j].x, nd[j], pol_keep);
                            }
                            tried[j] = true;
                        }
                    }
                }
#pragma unroll
                for (int j = 0; j < EPT; ++j) {
                    push[j] = tried[j] && nd[j] < old[j];
                    if (push[j] && p.filt) st_filt(p.filt + a[j].x, filt_enc(nd[j], p.filt_shift));
                }
#pragma unroll
                for (int j = 0; j < EPT; ++j) {
                    if (!__any_sync(FULL, push[j])) continue;
                    const unsigned o = push[j] ? bucket_of<kF>((unsigned long long)nd[j], k, hd.h, p.nb) : 0u;
                    const bool kept = keep(push[j] && o == 0, a[j].x, (unsigned long long)nd[j], false, 0ull, 0u);
                    emit(push[j] && !kept, a[j].x, (unsigned long long)nd[j], o);
                }
            };
            // The same round for the common case of the throughput build (gathered filter, no
            // 16-bit filter): the gathers and REDs are predicated instructions, not branches,
            // and the per-arc tests of the other cases are compiled out of the loop.
            auto body_fire = [&](const unsigned base, const DistT (&dv)[EPT], const uint2 (&a)[EPT]) {
                DistT nd[EPT], cur[EPT];
                bool ok[EPT], push[EPT];
                bool anybad = false;
#pragma unroll
                for (int j = 0; j < EPT; ++j) {
                    const bool lv = base + j * 32 + lane < we;
                    bool bd;
                    nd[j] = relax_narrow<kF, DistT>(dv[j], a[j].y, bd);
                    anybad |= lv && bd;
                    ok[j] = lv && !bd;
                }
#pragma unroll
                for (int j = 0; j < EPT; ++j) cur[j] = ld_keep_if(ok[j], p.dist + a[j].x, pol_keep);
                if (!kF && anybad) atomicOr(&p.ctl->status, kStDistOverflow);  // 32-bit distances insufficient
#pragma unroll
                for (int j = 0; j < EPT; ++j) {  // (cur = 0 where !ok: no push)
                    push[j] = nd[j] < cur[j];
                    red_min_keep_if(push[j], p.dist + a[j].x, nd[j], pol_keep);
                }
#pragma unroll
                for (int j = 0; j < EPT; ++j) {
                    if (!__any_sync(FULL, push[j])) continue;
                    unsigned o;
                    if constexpr (kTP) {  // 32-bit distances: the bucket in 32-bit arithmetic
                        const unsigned jb = k >= 32u ? 0u : (unsigned)nd[j] >> k;
                        o = jb <= h32 ? 0u : min(jb - h32, nbm);
                    } else {
                        o = push[j] ? bucket_of<kF>((unsigned long long)nd[j], k, hd.h, p.nb) : 0u;
                    }
                    const bool kept = keep(push[j] && o == 0, a[j].x, (unsigned long long)nd[j], false, 0ull, 0u);
                    emit(push[j] && !kept, a[j].x, (unsigned long long)nd[j], o);
                }
            };
            auto stream = [&](auto&& round) {
                if (PIPE && we > wb + kChunk) {
                    // software pipeline: round r+1's owners and arc loads are issued before
                    // round r's gathers and atomics
                    DistT dv_n[EPT];
                    uint2 a_n[EPT];
                    if (wb < we) fetch(wb, dv_n, a_n);
                    for (unsigned base = wb; base < we;) {
                        DistT dv[EPT];
                        uint2 a[EPT];
#pragma unroll
                        for (int j = 0; j < EPT; ++j) {
                            dv[j] = dv_n[j];
                            a[j] = a_n[j];
                        }
                        const unsigned nxt = base + kChunk;
                        if (nxt < we) fetch(nxt, dv_n, a_n);
                        round(base, dv, a);
                        base = nxt;
                    }
                } else {
                    for (unsigned base = wb; base < we; base += kChunk) {
                        DistT dv[EPT];
                        uint2 a[EPT];
                        fetch(base, dv, a);
                        round(base, dv, a);
                    }
                }
            };
            if constexpr (!WLC) {
                if (fire) stream(body_fire);
                else stream(body);
            } else {
                stream(body);
            }
            // ------------------------------------------------ warp-local continuation
            // Latency regime only (road-like graphs: a few hundred items per bucket,
            // thousands of dependent hops).  The warp pops up to 32 of its own kept
            // children (one per lane, LIFO), re-checks staleness while loading the row,
            // relaxes each child's arcs EPT at a time with no filter load, and keeps /
            // emits the improved ones exactly like the batch does -- one hop costs three
            // dependent L2 round trips (row, arcs, atomicMin) and no CTA barrier.  The
            // children are covered by this batch's own pending count (the batch
            // completes after its warps' queues drain), so no counter is touched.
            // Rows longer than kWDeg go back through the ring (head bucket).
            constexpr unsigned kWDeg = 8u * EPT;
            if constexpr (WLC) while (wq_n > 0) {
                __syncwarp();  // the queue entries written by other lanes (keep) are visible
                const unsigned take = wq_n < 32u ? wq_n : 32u;
                const unsigned st0 = wq_h;  // logical start of this hop's items
                const unsigned ph = wq0 + (st0 + lane) % kWQ;
                const bool has = lane < (int)take;
                unsigned v = 0, deg = 0;
                unsigned long long dv = kInf, b = 0;
                if (has) {
                    v = s_wqv[ph];
                    dv = (unsigned long long)s_wqd[ph];
                    b = s_wqb[ph];
                    deg = s_wqn[ph];
                }
                __syncwarp();
                wq_n -= take;
                wq_h += take;
                // long rows go back to the head bucket through the ring (their popper
                // re-checks staleness)
                const bool big = has && deg > kWDeg;
                emit(big, v, dv, 0u);
                bool lv = has && !big;
                // the stale re-check is in flight together with the first arc loads (one
                // round trip); skipping it expands superseded children (measured 1.7x ->
                // 3.2x work on ROAD)
                const unsigned long long cur = lv ? (unsigned long long)ld_keep(p.dist + v, pol_keep) : 0ull;
                uint2 a[EPT];
#pragma unroll
                for (int j = 0; j < EPT; ++j)
                    a[j] = lv && (unsigned)j < deg ? ld_stream_u2(p.adj + b + j, pol_stream) : make_uint2(0u, 0u);
                lv = lv && cur >= dv;
                // first-expansion bit for the controller: the atomicOr's result is consumed
                // only after this hop's relaxations are issued (waiting for it here put a third
                // dependent round trip into every hop of the dynamic mode)
                unsigned fword = 0, fbit = 0;
                if (lv && p.dynamic) {
                    fbit = 1u << (v & 31);
                    fword = atomicOr(p.expanded + (v >> 5), fbit);
                }
                if (!lv) deg = 0;
                const unsigned nl = (unsigned)__popc(__ballot_sync(FULL, lv));
                const unsigned ns = (unsigned)__popc(__ballot_sync(FULL, has && !lv && !big));
                const unsigned sumdeg = __reduce_add_sync(FULL, deg);
                const unsigned maxdeg = __reduce_max_sync(FULL, deg);
                if (lane == 0) {
                    if (nl) atomicAdd(&s_wst[0], nl);
                    if (sumdeg) atomicAdd(&s_wst[2], sumdeg);
                    if (ns) atomicAdd(&s_wst[3], ns);
                }
                for (unsigned kk = 0; kk < maxdeg; kk += EPT) {
                    if (kk > 0) {
#pragma unroll
                        for (int j = 0; j < EPT; ++j)
                            a[j] = kk + j < deg ? ld_stream_u2(p.adj + b + kk + j, pol_stream) : make_uint2(0u, 0u);
                    }
                    unsigned long long nd[EPT], rb[EPT], re[EPT];
                    DistT old[EPT];
                    bool push[EPT];
#pragma unroll
                    for (int j = 0; j < EPT; ++j) {
                        push[j] = false;
                        old[j] = (DistT)0;
                        rb[j] = re[j] = 0;
                        nd[j] = kk + j < deg ? relax_sum<kF>(dv, a[j].y) : kInf;
                        if (kk + j < deg) {
                            if (sum_unusable<kF>(nd[j], kInf)) {
                                if (!kF) atomicOr(&p.ctl->status, kStDistOverflow);
                            } else {
                                // the target's row is fetched in the same round trip as the
                                // atomicMin: a kept child starts its hop with its arc loads
                                old[j] = atomic_min_keep(p.dist + a[j].x, (DistT)nd[j], pol_keep);
                                rb[j] = ld_stream_u64(p.off + a[j].x, pol_stream);
                                re[j] = ld_stream_u64(p.off + a[j].x + 1, pol_stream);
                                push[j] = true;
                            }
                        }
                    }
#pragma unroll
                    for (int j = 0; j < EPT; ++j) {
                        push[j] = push[j] && nd[j] < (unsigned long long)old[j];
                        if (push[j] && p.filt) st_filt(p.filt + a[j].x, filt_enc(nd[j], p.filt_shift));
                        if (!__any_sync(FULL, push[j])) continue;
                        const unsigned o = push[j] ? bucket_of<kF>(nd[j], k, hd.h, p.nb) : 0u;
                        const bool kept = keep(push[j] && o == 0, a[j].x, nd[j], true, rb[j], (unsigned)(re[j] - rb[j]));
                        emit(push[j] && !kept, a[j].x, nd[j], o);
                    }
                }
                const unsigned nf = (unsigned)__popc(__ballot_sync(FULL, fbit != 0 && (fword & fbit) == 0));
                if (lane == 0 && nf) atomicAdd(&s_wst[1], nf);
            }
            rank_segment();  // bucket ranks of this warp's staged pushes, before the CTA flush
        }
        if constexpr (CA) {
            // the batch's claim state (s_got/s_slot/s_idx/s_head/s_task) was consumed before
            // the streaming barrier
            // the first warp to finish its slice claims (its round trips overlap the slower
            // warps' streaming instead of extending the batch when warp 0 is the last;
            // ER -1.7 %, RMAT -0.7 %, sweeps r02 §10)
            // A batch that keeps children (lcap != 0) claims ahead too: its kept children run
            // first (loop top), the claimed batch waits in s_got.. until no local batch is left
            // (one claim ahead at most; kept children use their own slot, kslot)
            bool claimer = false;
            if (!s_ahead) {
                unsigned f = 0;
                if (lane == 0) f = atomicAdd(&s_fin, 1u);
                claimer = __shfl_sync(FULL, f, 0) == 0;
            }
            if (claimer) {
                unsigned sl = 0, st = 0;
                unsigned long long idx = 0;
                Head hd2;
                bool tk;
                const unsigned g = claim_batch<DistT, BT, !WLC>(p, lane, sl, idx, hd2, st, tk);
                if (lane == 0 && g) {
                    s_got = g;
                    s_slot = sl;
                    s_idx = idx;
                    s_head = hd2;
                    s_task = tk ? 1u : 0u;
                    s_ahead = 1;
                    backoff = 0;
                }
            }
        }
        // first expansions of this batch's pops (controller), one shared atomic per warp
        {
            const unsigned nf = (unsigned)__popc(__ballot_sync(FULL, fbit != 0 && (fword & fbit) == 0));
            if (lane == 0 && nf) atomicAdd(&s_nf, nf);
        }
        // End of batch, three barriers at most: B1 (streaming done: staging, s_lnext, s_nf, the
        // claim-ahead and the warp-local counters are final), B2 (reserves done), B3 (stores
        // done).  No barrier closes the batch: warp 0 publishes, completes and runs the
        // controller while the other warps start the next batch's pop (they meet again at its
        // first barrier); what they read here was written before B1 and is reset only after
        // that next barrier (s_lnext) or by thread 0 itself (s_total, s_direct, s_fin, s_nf).
        const bool any_staged = __syncthreads_or(wfill != 0) != 0;  // B1
        const unsigned kept = s_lnext < lcap ? s_lnext : lcap;
        unsigned total = 0;
        if (any_staged) {
            // ---------------------------------------------------- flush to the ring
            const long long tf = prof ? clock64() : 0;
            {
                // column scan of s_wcnt over the warps, all warps at once: lanes form
                // segments of kWarps (one per bucket), lane w%kWarps = warp w's count;
                // the segment's last lane holds the CTA's count for the bucket and
                // reserves it (returning atomic: the reserve, which also counts the
                // children for termination, precedes this CTA's completion release)
                constexpr unsigned kBPW = kWarps >= 32 ? 1u : 32u / kWarps;  // buckets per warp
                const unsigned o = (unsigned)warp * kBPW + (unsigned)lane / kWarps;
                const unsigned w = (unsigned)lane % kWarps;
                const bool mine = o < p.nb;
                const unsigned v = mine ? s_wcnt[w][o] : 0u;
                unsigned x = v;
#pragma unroll
                for (unsigned d = 1; d < (unsigned)kWarps; d <<= 1) {
                    const unsigned y = __shfl_up_sync(FULL, x, d, kWarps);
                    if (w >= d) x += y;
                }
                if (mine) s_wcnt[w][o] = x - v;  // warp w's offset inside the CTA's reservation
                if (mine && w == (unsigned)kWarps - 1) {
                    s_cnt[o] = x;
                    if (x) {
                        atomicAdd(&s_total, x);
                        const unsigned long long b = atomicAdd(&p.bk[(hs + o) & nbm].reserve.v, (unsigned long long)x);
                        SSSP_FUZZ_AT(FZ_RESERVE);
                        s_base[o] = b;
                        if (flat_overflow(p, b, x, chk)) atomicOr(&p.ctl->status, kStRingOverflow);  // no laps (D13)
                        chunks_for_range(p, (hs + o) & nbm, b, x, chk);
                        if (chk) {  // the range's chunks, once, for every store below
                            for (unsigned q = 0; q < kFlushChunks; ++q) {
                                const unsigned long long ci = (b >> kChunkShift) + q;
                                s_cid[o][q] = (ci << kChunkShift) < b + x ? chunk_of(p, (hs + o) & nbm, ci << kChunkShift) : 0u;
                            }
                        }
                        if (p.dynamic && o == nbm) atomicAdd(&p.ctl->g_clip, (unsigned long long)x);
                    }
                }
            }
            __syncthreads();  // B2
            total = s_total;
            // each warp stores its own segment (coalesced runs per bucket)
            for (unsigned i = lane; i < wfill; i += 32) {
                const unsigned my = (unsigned)warp * kSeg + i;
                const unsigned o = s_soff[my];
                const unsigned sl = (hs + o) & nbm;
                const unsigned long long idx = s_base[o] + s_wcnt[warp][o] + s_rank[my];
                SSSP_FUZZ_AT(FZ_PUBLISH);
                // the slot's one writer this run (D13); beyond cap the run is aborted
                if (chk) {
                    const unsigned id1 = s_cid[o][(idx >> kChunkShift) - (s_base[o] >> kChunkShift)];
                    if (id1) IT::store(chunk_item(p, id1, idx), s_items[my]);
                } else if (idx < p.cap) {
                    IT::store(item_ptr(p, sl, idx, chk), s_items[my]);
                }
            }
            __syncwarp();
            if (lane < (int)p.nb) s_wcnt[warp][lane] = 0;  // this warp's row is no longer read
            __syncthreads();  // B3
            if (warp == 0 && lane < (int)p.nb) {
                const unsigned c = s_cnt[lane];
                if (p.dynamic && lane == 0) atomicAdd(&p.ctl->g_push, (unsigned long long)(total + s_direct));
                if (c) {
                    atomicAdd(&p.bk[(hs + lane) & nbm].avail.v, (unsigned long long)c);  // publish
                    s_cnt[lane] = 0;
                }
            }
            if (prof) {
                tq += clock64() - tf;
                s_prof[PR_N_FLUSH] += 1;
            }
        }
        if (prof) {
            const long long t1 = clock64();
            s_prof[PR_ROUNDS] += t1 - t0 - tq - tw;
            s_prof[PR_FLUSH] += tq;
            s_prof[PR_WINDOW] += tw;
            t0 = t1;
        }

        // ------------------------------------------------------------ complete
        // (thread 0 alone reads and resets the CTA's shared counters)
        unsigned w_exp = 0, w_first = 0, w_kept = 0, nfirst = 0;
        if (tid == 0) {
            const unsigned direct = s_direct;
            if (!any_staged && p.dynamic && direct) atomicAdd(&p.ctl->g_push, (unsigned long long)direct);
            c_push += total + direct;
            s_total = 0;
            s_direct = 0;
            s_fin = 0;
            nfirst = s_nf;
            s_nf = 0;
            w_exp = s_wst[0];
            w_first = s_wst[1];
            w_kept = s_wst[4];
            if (wlc) {
                c_vert += w_exp;
                c_edges += s_wst[2];
                c_stale += s_wst[3];
                c_push += s_wst[4];
                c_local += s_wst[4];
                s_wst[0] = s_wst[1] = s_wst[2] = s_wst[3] = s_wst[4] = 0;
            }
            // one atomic: the kept children inherit the parents' accounting; a completion
            // is a release (common.cuh red_release_add_u64): the children's reserve
            // atomics (warp flushes before B1, the CTA flush before B2) are ordered before
            // it by the CTA barriers
            SSSP_FUZZ_AT(FZ_COMPLETE);
            if (got > kept) red_release_add_u64(&p.bk[slot].done.v, (unsigned long long)(got - kept));
            else if (kept > got) atomicAdd(&p.bk[slot].local.v, (unsigned long long)(kept - got));
            c_push += kept;
            c_local += kept;
        }
        if (p.dynamic && warp == 0) {
            unsigned run_ctl = 0;
            if (lane == 0) {
                if (nexp + w_exp) {
                    atomicAdd(&p.ctl->g_exp, (unsigned long long)(nexp + w_exp));
                    atomicAdd(&p.ctl->g_first, (unsigned long long)(nfirst + w_first));
                }
                if (kept + w_kept) atomicAdd(&p.ctl->g_push, (unsigned long long)(kept + w_kept));
                const unsigned long long now = globaltimer();
                const unsigned long long last = ld_relaxed_u64(&p.ctl->last_ctl_ns);
                if (now - last > p.period_ns && atomicCAS(&p.ctl->last_ctl_ns, last, now) == last) run_ctl = 1;
            }
            if (__shfl_sync(FULL, run_ctl, 0)) periodic_step<DistT>(p, lane);
        }
        have_local = kept;
        kslot = slot;
        if (prof) s_prof[PR_COMPLETE] += clock64() - t0;
    }

    if (tid == 0) {
        atomicAdd(&p.ctl->st_vertices, c_vert);
        atomicAdd(&p.ctl->st_edges, c_edges);
        atomicAdd(&p.ctl->st_pushes, c_push);
        atomicAdd(&p.ctl->st_stale, c_stale);
        atomicAdd(&p.ctl->st_local, c_local);
        if (p.prof) {
            s_prof[PR_TOTAL] = clock64() - t_begin;
            s_prof[PR_N_CTAS] = 1;
            for (int i = 0; i < (int)kProfCounters; ++i) atomicAdd(&p.ctl->prof[i], s_prof[i]);
        }
    }
}

}  // namespace adds

// common.cuh -- device data structures and PTX helpers of the ADDS worklist.
//
// Layout in HBM:
//   BucketCtl[32]  per ring slot: reserve (P:159 resv_ptr), avail (published -
//                  claimed gate), claim (P:159 read_ptr), done (P:176 CWC),
//                  local (children kept CTA-local);
//                  every counter on its own 128-B line so the L2 atomic units
//                  of different counters never serialise on one line.
//   Ctl            head state (16 B, 128-bit CAS), status bits, statistics,
//                  trace cursor, phase profile.
//   ring           nb circular arrays of C items each (pre-allocated).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace adds {

constexpr uint32_t kMaxBuckets = 32;

// status bits written by the device
constexpr unsigned kStRingOverflow = 1u;   // a bucket's circular array would lap an unclaimed item
constexpr unsigned kStDistOverflow = 2u;   // 32-bit distance would overflow -> rerun with 64-bit
constexpr unsigned kStTimeout = 4u;        // watchdog
constexpr unsigned kStBug = 8u;            // internal invariant violated

// Phase profile (SSSP_FLAG_PROFILE), summed over CTAs; see sssp_get_profile().
enum ProfIdx {
    PR_CLAIM = 0, PR_IDLE, PR_POP, PR_SCAN, PR_ROUNDS, PR_FLUSH, PR_COMPLETE, PR_TOTAL,
    PR_N_RING, PR_N_LOCAL, PR_N_IDLE, PR_N_FLUSH, PR_N_ROUND, PR_N_CTAS, PR_WINDOW, PR_N_WINDOW,
    kProfCounters = 16
};

struct alignas(128) Counter {
    unsigned long long v;
    unsigned long long pad_[15];
};

struct BucketCtl {
    Counter reserve;  // items reserved by writers (monotone)      = resv_ptr
    Counter avail;    // signed: published and not yet claimed      (claim gate)
    Counter claim;    // items claimed by workers (monotone)        = read_ptr
    Counter done;     // items whose processing completed           = CWC
    Counter local;    // items kept CTA-local (never stored in the ring) charged to this bucket
};
// Hub-split chunk (§8(a) A5): arcs [beg, beg + len) of vertex v expanded at
// distance d, charged to ring slot `slot` (its `local` counter was raised when the
// chunk was made; completing the chunk raises `done`).  len == 0 marks an empty
// entry: the producer stores the payload, fences, then stores len; the consumer
// spins on len (acquire), reads, and clears it.  Queue counters live in
// BucketCtl[kSplitQ] (reserve / avail / claim, the bucket-ring protocol).
struct alignas(32) SplitTask {
    unsigned long long beg;
    unsigned long long d;
    unsigned v;
    unsigned len;
    unsigned slot;
    unsigned pad_;
};
constexpr uint32_t kSplitQ = kMaxBuckets;

// Chunked bucket storage (SSSP_FLAG_CHUNKED_RING; the paper's block pool): the
// buckets' index spaces map through per-bucket chunk tables onto a shared pool of
// kChunkItems-item chunks.  The reserver whose range contains a chunk's first index takes
// the chunk (fresh, else from the free ring) and publishes it in the table; a chunk returns
// to the free ring when all its items have been read (and cleared), so memory is bounded by
// the items alive at once, not by the pushes of a run.
constexpr unsigned kChunkShift = 12;
constexpr unsigned kChunkItems = 1u << kChunkShift;
struct ChunkPool {
    Counter fresh;     // never-used chunks handed out (bump allocator)
    Counter freserve;  // free-ring pushes (monotone)
    Counter favail;    // signed: freed chunks published and not yet taken
    Counter fclaim;    // free-ring pops (monotone)
};
// SplitTask.len states besides a real length: 0 = free, kLenBusy = a writer owns the
// slot (payload being written), kLenReading = a reader owns it (payload being read).
// Writers take a free slot by CAS 0 -> busy and publish with a release store of the
// length; readers take a published slot by CAS len -> reading and free it with a
// release store of 0 after reading, so no chunk is lost or taken twice even when
// the queue laps with chunks claimed but not yet read.
constexpr unsigned kLenBusy = 0xFFFFFFFFu;
constexpr unsigned kLenReading = 0xFFFFFFFEu;  // index of the split queue's counters
// In flight for bucket b = reserve + local - done.  The bucket is complete when
// that is 0, and the run is finished when every bucket is complete
// (exact quiescence, reading R11 of P:182): children are always counted (reserve
// or local) before their parent's completion is.

// Head state, updated only by 128-bit CAS (one writer per head switch).
//   h    : absolute number of the head bucket (units of Delta = 2^k)
//   meta : [0,8) hs = ring slot of the head  [8,16) k = log2 Delta
//          [16,24) A = active buckets        [24,32) floor of k (clip bound)
//          [32,48) controller steps / head switches since the last Delta change
//          [48,56) ceiling of k: a k found wasteful is not grown into again (0xff = none)
struct alignas(16) Head {
    unsigned long long h;
    unsigned long long meta;
};

__host__ __device__ __forceinline__ unsigned long long pack_meta(unsigned hs, unsigned k, unsigned A,
                                                                 unsigned flo, unsigned since, unsigned ceil = 0xffu,
                                                                 unsigned pk = 0u) {
    return (unsigned long long)(hs & 0xff) | ((unsigned long long)(k & 0xff) << 8) |
           ((unsigned long long)(A & 0xff) << 16) | ((unsigned long long)(flo & 0xff) << 24) |
           ((unsigned long long)(since & 0xffff) << 32) | ((unsigned long long)(ceil & 0xff) << 48) |
           ((unsigned long long)(pk & 0xff) << 56);
}
__host__ __device__ __forceinline__ unsigned meta_hs(unsigned long long m) { return (unsigned)(m & 0xff); }
__host__ __device__ __forceinline__ unsigned meta_k(unsigned long long m) { return (unsigned)((m >> 8) & 0xff); }
__host__ __device__ __forceinline__ unsigned meta_A(unsigned long long m) { return (unsigned)((m >> 16) & 0xff); }
__host__ __device__ __forceinline__ unsigned meta_floor(unsigned long long m) { return (unsigned)((m >> 24) & 0xff); }
__host__ __device__ __forceinline__ unsigned meta_since(unsigned long long m) { return (unsigned)((m >> 32) & 0xffff); }
__host__ __device__ __forceinline__ unsigned meta_ceil(unsigned long long m) { return (unsigned)((m >> 48) & 0xff); }
// [56,64) parked shrinks since the head last switched (bounds the shrink-without-head-switch rule)
__host__ __device__ __forceinline__ unsigned meta_pk(unsigned long long m) { return (unsigned)((m >> 56) & 0xff); }

struct TraceEntry {  // mirrors sssp_trace_entry
    unsigned long long time_ns, head, pending_total, pending_window, pending_tail;
    unsigned delta_log2, active;
    unsigned waste_permille, reason;  // reason: 1 head switch, 2 periodic step
};

struct alignas(128) Ctl {
    Head head;
    char pad0_[128 - sizeof(Head)];
    unsigned status;
    unsigned trace_count;
    unsigned head_switches;
    unsigned delta_changes;
    unsigned long long t_start;  // %globaltimer at init (watchdog)
    char pad2_[104];
    // Delta-controller work signal (own lines: updated with REDs once per batch)
    unsigned long long g_exp;     // items expanded (not stale)
    char pad4_[120];
    unsigned long long g_first;   // first expansions of a vertex (distinct vertices expanded)
    char pad5_[120];
    unsigned long long last_ctl_ns, exp_mark, first_mark;  // controller period / window start
    unsigned long long push_mark, clip_mark;
    char pad6_[88];
    unsigned long long g_push;    // items pushed (ring + kept)
    char pad7_[120];
    unsigned long long g_clip;    // items pushed into the tail bucket (clipped)
    char pad8_[120];
    unsigned long long g_busy;    // CTAs holding a batch (the paper's "work assigned")
    unsigned last_waste;          // last measured re-expansion share + 1 (0 = never measured)
    char pad9_[116];
    unsigned long long st_local;  // items continued CTA-locally
    // statistics (flushed once per CTA at exit, or by finalize)
    unsigned long long st_vertices, st_edges, st_pushes, st_stale;
    unsigned long long reach_v, reach_e, max_dist;
    unsigned long long pad3_[8];
    unsigned long long prof[kProfCounters];  // SSSP_FLAG_PROFILE: per-phase SM cycles / counts (sum over CTAs)
};
static_assert(sizeof(Ctl) % 128 == 0, "Ctl layout");

// ------------------------------------------------------------ PTX helpers
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ long long ld_relaxed_s64(const long long* p) {
    long long v;
    asm volatile("ld.relaxed.gpu.global.s64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_u32(unsigned* p, unsigned v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_u32(unsigned* p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned cas_acquire_u32(unsigned* p, unsigned cmp, unsigned val) {
    unsigned r;
    asm volatile("atom.acquire.gpu.global.cas.b32 %0, [%1], %2, %3;" : "=r"(r) : "l"(p), "r"(cmp), "r"(val) : "memory");
    return r;
}
__device__ __forceinline__ unsigned ld_relaxed_u32(const unsigned* p) {
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void ld_relaxed_v2u64(const void* p, unsigned long long& a, unsigned long long& b) {
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ void st_relaxed_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_v2u64(void* p, unsigned long long a, unsigned long long b) {
    asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
// dist loads go to L2 (.cg): dist is updated by L2 atomics, an L1-stale value is
// still a valid upper bound (it only weakens the filter) but L2 is fresher.
__device__ __forceinline__ unsigned ld_cg(const unsigned* p) { return __ldcg(p); }
__device__ __forceinline__ unsigned long long ld_cg(const unsigned long long* p) { return __ldcg(p); }

// ---- L2 residency (D5): the arc stream (GBs, read ~once) is marked
// evict_first so it cannot push the distance array (67/134 MB, gathered and
// atomically updated at random) out of the 126 MB L2; dist accesses are evict_last.
__device__ __forceinline__ unsigned long long policy_evict_first() {
    unsigned long long p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// evict_last residency is bounded by the L2 persisting set-aside
// (cudaLimitPersistingL2CacheSize); `frac` = set-aside / dist bytes keeps a
// stable subset of dist resident when it does not fit entirely.
__device__ __forceinline__ unsigned long long policy_evict_last(float frac) {
    unsigned long long p;
    asm volatile("createpolicy.fractional.L2::evict_last.L2::evict_unchanged.b64 %0, %1;" : "=l"(p) : "f"(frac));
    return p;
}
__device__ __forceinline__ uint2 ld_stream_u2(const uint2* a, unsigned long long pol) {
    uint2 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0, %1}, [%2], %3;"
                 : "=r"(r.x), "=r"(r.y) : "l"(a), "l"(pol));
    return r;
}
__device__ __forceinline__ uint2 ld_stream_u2_if(bool pr, const uint2* a, unsigned long long pol) {
    uint2 r = make_uint2(0u, 0u);
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %3, 0; @q ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0, %1}, [%2], %4; }"
                 : "+r"(r.x), "+r"(r.y) : "l"(a), "r"((unsigned)pr), "l"(pol));
    return r;
}
__device__ __forceinline__ unsigned long long ld_stream_u64(const unsigned long long* a, unsigned long long pol) {
    unsigned long long r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(r) : "l"(a), "l"(pol));
    return r;
}
__device__ __forceinline__ unsigned ld_keep(const unsigned* a, unsigned long long pol) {
    unsigned r;
    asm volatile("ld.global.cg.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(a), "l"(pol));
    return r;
}
__device__ __forceinline__ unsigned long long ld_keep(const unsigned long long* a, unsigned long long pol) {
    unsigned long long r;
    asm volatile("ld.global.cg.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(r) : "l"(a), "l"(pol));
    return r;
}
// 16-bit upper-bound filter of dist (D11)
__device__ __forceinline__ unsigned short ld_filt(const unsigned short* a) {
    unsigned short r;
    asm volatile("ld.global.cg.u16 %0, [%1];" : "=h"(r) : "l"(a));
    return r;
}
__device__ __forceinline__ void st_filt(unsigned short* a, unsigned short v) {
    asm volatile("st.global.cg.u16 [%0], %1;" ::"l"(a), "h"(v) : "memory");
}
__device__ __forceinline__ unsigned atomic_min_keep(unsigned* a, unsigned v, unsigned long long pol) {
    unsigned r;
    asm volatile("atom.global.L2::cache_hint.min.u32 %0, [%1], %2, %3;" : "=r"(r) : "l"(a), "r"(v), "l"(pol) : "memory");
    return r;
}
__device__ __forceinline__ unsigned long long atomic_min_keep(unsigned long long* a, unsigned long long v,
                                                              unsigned long long pol) {
    unsigned long long r;
    asm volatile("atom.global.L2::cache_hint.min.u64 %0, [%1], %2, %3;" : "=l"(r) : "l"(a), "l"(v), "l"(pol) : "memory");
    return r;
}

// fire-and-forget atomic min (RED: no result, no round trip for the issuing warp)
// Predicated forms for the throughput loop: the instruction carries the predicate, so the
// compiler emits no branch / reconvergence pair around it (one per arc otherwise).
__device__ __forceinline__ unsigned ld_keep_if(bool pr, const unsigned* a, unsigned long long pol) {
    unsigned r = 0u;
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %2, 0; @q ld.global.cg.L2::cache_hint.u32 %0, [%1], %3; }"
                 : "+r"(r) : "l"(a), "r"((unsigned)pr), "l"(pol));
    return r;
}
__device__ __forceinline__ unsigned long long ld_keep_if(bool pr, const unsigned long long* a, unsigned long long pol) {
    unsigned long long r = 0ull;
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %2, 0; @q ld.global.cg.L2::cache_hint.u64 %0, [%1], %3; }"
                 : "+l"(r) : "l"(a), "r"((unsigned)pr), "l"(pol));
    return r;
}
__device__ __forceinline__ void red_min_keep_if(bool pr, unsigned* a, unsigned v, unsigned long long pol) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %3, 0; @q red.global.L2::cache_hint.min.u32 [%0], %1, %2; }"
                 ::"l"(a), "r"(v), "l"(pol), "r"((unsigned)pr) : "memory");
}
__device__ __forceinline__ void red_min_keep_if(bool pr, unsigned long long* a, unsigned long long v,
                                                unsigned long long pol) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %3, 0; @q red.global.L2::cache_hint.min.u64 [%0], %1, %2; }"
                 ::"l"(a), "l"(v), "l"(pol), "r"((unsigned)pr) : "memory");
}
__device__ __forceinline__ void red_min_keep(unsigned* a, unsigned v, unsigned long long pol) {
    asm volatile("red.global.L2::cache_hint.min.u32 [%0], %1, %2;" ::"l"(a), "r"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void red_min_keep(unsigned long long* a, unsigned long long v, unsigned long long pol) {
    asm volatile("red.global.L2::cache_hint.min.u64 [%0], %1, %2;" ::"l"(a), "l"(v), "l"(pol) : "memory");
}

__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// Completion counter update with gpu-scope release semantics: every write of the
// CTA that precedes it (children's reserve atomics and ring stores, ordered by the
// CTA barrier) is visible to whoever acquire-reads the counter and sees the
// increment (try_advance / bucket_pending read `done` with ld.acquire before
// `reserve` and `local`), so a bucket can never look complete while one of its
// items' children is not yet counted (exact termination).
__device__ __forceinline__ void red_add_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_release_add_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// ---- schedule fuzzing (libsssp_fuzz.so, built with -DSSSP_FUZZ; tests only).
// A hash of the SM clock, the global timer, the CTA, the thread and the site picks
// one call in four and sleeps 32 ns .. 4 us there, so the worklist protocol is
// exercised under reorderings the natural schedule rarely produces: a reserved
// slot published late, a claim separated from its read_ptr update, a completion
// or a head advance delayed past other CTAs' work.
enum FuzzSite : unsigned { FZ_CLAIM = 1, FZ_POP, FZ_RESERVE, FZ_PUBLISH, FZ_COMPLETE, FZ_HEAD, FZ_CHUNK };
#ifdef SSSP_FUZZ
__device__ __forceinline__ void fuzz_delay(unsigned site) {
    const unsigned long long t = globaltimer() ^ ((unsigned long long)clock64() << 7);
    unsigned h = (unsigned)(t ^ (t >> 32)) * 0x9E3779B1u;
    h ^= blockIdx.x * 0x85EBCA6Bu ^ threadIdx.x * 0xC2B2AE35u ^ site * 0x27D4EB2Fu;
    h ^= h >> 15;
    h *= 0x2C1B3C6Du;
    h ^= h >> 12;
    h *= 0x297A2D39u;
    h ^= h >> 15;
    if ((h & 3u) == 0u) __nanosleep(32u + ((h >> 4) & 4095u));
}
#define SSSP_FUZZ_AT(site) ::adds::fuzz_delay(site)
#else
#define SSSP_FUZZ_AT(site) ((void)0)
#endif

// 128-bit CAS on the head state (sm_90+: atom.cas.b128).
__device__ __forceinline__ bool cas_head(Head* addr, Head expect, Head desired, Head& seen) {
    unsigned long long o0, o1;
    asm volatile(
        "{\n\t.reg .b128 d, b, c;\n\t"
        "mov.b128 b, {%2, %3};\n\t"
        "mov.b128 c, {%4, %5};\n\t"
        "atom.relaxed.gpu.global.cas.b128 d, [%6], b, c;\n\t"
        "mov.b128 {%0, %1}, d;\n\t}"
        : "=l"(o0), "=l"(o1)
        : "l"(expect.h), "l"(expect.meta), "l"(desired.h), "l"(desired.meta), "l"(addr)
        : "memory");
    seen.h = o0;
    seen.meta = o1;
    return o0 == expect.h && o1 == expect.meta;
}

__device__ __forceinline__ Head ld_head(const Head* p) {
    Head h;
    ld_relaxed_v2u64(p, h.h, h.meta);
    return h;
}

// 8-byte asynchronous global->shared copy (LDGSTS), streamed through L2 (evict_first).
// `sdst` is a shared-window address (convert the base once with smem_addr()).
__device__ __forceinline__ unsigned smem_addr(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void cp_async_8(unsigned sdst, const void* gsrc, unsigned long long pol) {
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 8, %2;" ::"r"(sdst), "l"(gsrc), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// non-blocking L2 prefetch (no register result, nothing waits on it)
__device__ __forceinline__ void prefetch_l2(const void* p) {
    asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(p));
}

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// ------------------------------------------------------------ item formats
// Ring slot protocol (D13).  Claims hand out ring indices in order but
// items are published out of order (the avail gate counts items, not indices), so
// if a bucket's circular array lapped during a run, one slot could be targeted by
// the writers -- and the readers -- of two laps at once, and plain stores/loads
// could lose or duplicate an item.  The bucket arrays therefore never lap within
// a run: a reserve that would pass the capacity aborts the run as an overflow
// (the host doubles the array and re-runs), so every slot has exactly one writer
// and one reader per run and holds the empty marker at every run's start (a
// completed run reads and clears every slot it wrote; an aborted one is wiped).
// Then the item's own store is its publication and a plain load + clearing
// store its consumption.  take()/put() below are the lap-safe alternatives
// (exchange / CAS); they measured 6-7 % slower on RMAT/ER and are unused.
template <typename DistT>
struct ItemT;

template <>
struct ItemT<uint32_t> {
    using Raw = unsigned long long;
    static constexpr int kBytes = 8;
    __device__ __forceinline__ static Raw make(uint32_t v, unsigned long long d) {
        return (unsigned long long)v | (d << 32);
    }
    __device__ __forceinline__ static bool load(const void* slot, uint32_t& v, unsigned long long& d) {
        unsigned long long x = ld_relaxed_u64((const unsigned long long*)slot);
        v = (uint32_t)x;
        d = x >> 32;
        return x != ~0ull;
    }
    __device__ __forceinline__ static bool empty(const void* slot) {
        return ld_relaxed_u64((const unsigned long long*)slot) == ~0ull;
    }
    __device__ __forceinline__ static void store(void* slot, Raw r) { st_relaxed_u64((unsigned long long*)slot, r); }
    __device__ __forceinline__ static void clear(void* slot) { st_relaxed_u64((unsigned long long*)slot, ~0ull); }
    // Ownership-transferring ring ops (see "Ring slot protocol" above): take() empties
    // the slot with one exchange and owns whatever it returned; put() fills an empty
    // slot with one CAS.  Two writers of different laps, or two readers of different
    // laps, can therefore never both succeed on one slot.
    // (the claimer usually finds its item already there: exchange first, one round
    // trip; an exchange of empty with empty is harmless; spin on plain loads after)
    __device__ __forceinline__ static bool take(void* slot, uint32_t& v, unsigned long long& d, bool first) {
        if (!first && ld_relaxed_u64((const unsigned long long*)slot) == ~0ull) return false;
        const unsigned long long x = atomicExch((unsigned long long*)slot, ~0ull);
        v = (uint32_t)x;
        d = x >> 32;
        return x != ~0ull;
    }
    __device__ __forceinline__ static bool put(void* slot, Raw r) {
        return atomicCAS((unsigned long long*)slot, ~0ull, r) == ~0ull;
    }
};

template <>
struct ItemT<unsigned long long> {
    struct Raw {
        unsigned long long v, d;
    };
    static constexpr int kBytes = 16;
    __device__ __forceinline__ static Raw make(uint32_t v, unsigned long long d) { return Raw{v, d}; }
    __device__ __forceinline__ static bool load(const void* slot, uint32_t& v, unsigned long long& d) {
        unsigned long long a, b;
        ld_relaxed_v2u64(slot, a, b);
        v = (uint32_t)a;
        d = b;
        return a != ~0ull && b != ~0ull;
    }
    __device__ __forceinline__ static bool empty(const void* slot) {
        unsigned long long a, b;
        ld_relaxed_v2u64(slot, a, b);
        return a == ~0ull && b == ~0ull;
    }
    __device__ __forceinline__ static void store(void* slot, Raw r) { st_relaxed_v2u64(slot, r.v, r.d); }
    __device__ __forceinline__ static void clear(void* slot) { st_relaxed_v2u64(slot, ~0ull, ~0ull); }
    __device__ __forceinline__ static bool take(void* slot, uint32_t& v, unsigned long long& d, bool first) {
        unsigned long long a, b;
        if (!first) {
            ld_relaxed_v2u64(slot, a, b);
            if (a == ~0ull && b == ~0ull) return false;  // empty (a put is one 128-bit CAS)
        }
        asm volatile(
            "{\n\t.reg .b128 d, x;\n\t"
            "mov.b128 x, {%2, %3};\n\t"
            "atom.relaxed.gpu.global.exch.b128 d, [%4], x;\n\t"
            "mov.b128 {%0, %1}, d;\n\t}"
            : "=l"(a), "=l"(b)
            : "l"(~0ull), "l"(~0ull), "l"(slot)
            : "memory");
        v = (uint32_t)a;
        d = b;
        return !(a == ~0ull && b == ~0ull);
    }
    __device__ __forceinline__ static bool put(void* slot, Raw r) {
        unsigned long long o0, o1;
        asm volatile(
            "{\n\t.reg .b128 d, b, c;\n\t"
            "mov.b128 b, {%2, %3};\n\t"
            "mov.b128 c, {%4, %5};\n\t"
            "atom.relaxed.gpu.global.cas.b128 d, [%6], b, c;\n\t"
            "mov.b128 {%0, %1}, d;\n\t}"
            : "=l"(o0), "=l"(o1)
            : "l"(~0ull), "l"(~0ull), "l"(r.v), "l"(r.d), "l"(slot)
            : "memory");
        return o0 == ~0ull && o1 == ~0ull;
    }
};

template <typename DistT>
struct DistInf;
template <>
struct DistInf<uint32_t> {
    static constexpr uint32_t value = 0xFFFFFFFFu;
};
template <>
struct DistInf<unsigned long long> {
    static constexpr unsigned long long value = ~0ull;
};

}  // namespace adds

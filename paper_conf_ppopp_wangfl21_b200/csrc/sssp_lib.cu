// sssp_lib.cu -- the C ABI of include/sssp.h: handle, validation, options,
// workspace, launch sequence, status handling and retry.  All compute runs in
// the kernels of adds_kernel.cuh / aux_kernels.cuh; there is no CPU fallback.
#include <cuda_runtime.h>
#include <cub/cub.cuh>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <string>
#include <type_traits>
#include <vector>
#include <thread>
#include <chrono>

#include "../../include/sssp.h"
#include "adds_kernel.cuh"
#include "aux_kernels.cuh"
#include "certify_kernels.cuh"
#include "nearfar_kernel.cuh"
#include "bucket_map.h"

using namespace adds;

static_assert(sizeof(TraceEntry) == sizeof(sssp_trace_entry), "trace layout");

namespace {

thread_local std::string g_err;

sssp_status fail(sssp_status st, const std::string& msg) {
    g_err = msg;
    return st;
}

sssp_status cuda_fail(cudaError_t e, const char* what) {
    cudaGetLastError();  // clear sticky-free errors
    if (e == cudaErrorMemoryAllocation) return fail(SSSP_ERR_OUT_OF_MEMORY, std::string(what) + ": out of device memory");
    return fail(SSSP_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

#define CK(call, what)                                   \
    do {                                                 \
        cudaError_t e_ = (call);                         \
        if (e_ != cudaSuccess) return cuda_fail(e_, what); \
    } while (0)

unsigned long long next_pow2(unsigned long long x) {
    unsigned long long p = 1;
    while (p < x) p <<= 1;
    return p;
}
unsigned ilog2_round(double x) {
    if (!(x > 1.0)) return 0;
    double l = std::log2(x);
    long r = std::lround(l);
    return r < 0 ? 0u : (unsigned)r;
}

struct DevBuf {
    void* p = nullptr;
    size_t bytes = 0;
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        bytes = 0;
    }
};

}  // namespace

// One run's device state: a graph handle owns one workspace per concurrently
// running source (NEXT-1); workspace 0 runs on the caller's stream.
struct Workspace {
    DevBuf dist;        // 8n bytes (serves 32- and 64-bit distances)
    DevBuf ring;        // nb * cap * item bytes
    DevBuf bk, ctl, trace, expanded;
    DevBuf tasks;                   // hub-split chunk queue (SplitTask[tcap])
    DevBuf filt;                    // n x u16 upper-bound filter of dist (D11)
    // chunked bucket storage (SSSP_FLAG_CHUNKED_RING): ring = pool_chunks chunks of kChunkItems
    DevBuf ctab, chunk_used, free_ring, pool;
    bool chunked = false;
    unsigned pool_chunks = 0;
    unsigned long long tcap = 0;
    unsigned long long cap = 0;
    int ring_item_bytes = 0;
    unsigned trace_alloc = 0;
    Ctl* h_ctl = nullptr;  // pinned status block (mapped: written by status_copy_kernel)
    Ctl* h_ctl_dev = nullptr;  // its device alias
    cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
    cudaStream_t own_stream = nullptr;  // slots > 0
    // host dist_out batches: two device staging rows per slot and the events of their host copies
    DevBuf stage[2];
    cudaEvent_t cev[2] = {nullptr, nullptr};
    DevBuf nf_piles, nf_cnt;            // Near-Far ablation: 4 pile buffers + counters
    unsigned long long nf_cap = 0;
    int nf_item_bytes = 0;
    uint32_t last_grid = 0, last_block = 0, last_k0 = 0, last_worker = 0;
    void release() {
        dist.release();
        ring.release();
        bk.release();
        ctl.release();
        trace.release();
        expanded.release();
        tasks.release();
        filt.release();
        ctab.release();
        chunk_used.release();
        free_ring.release();
        pool.release();
        nf_piles.release();
        nf_cnt.release();
        if (h_ctl) cudaFreeHost(h_ctl);
        h_ctl = nullptr;
        for (auto& e : ev)
            if (e) cudaEventDestroy(e);
        if (own_stream) cudaStreamDestroy(own_stream);
        own_stream = nullptr;
        for (int b = 0; b < 2; ++b) {
            stage[b].release();
            if (cev[b]) cudaEventDestroy(cev[b]);
            cev[b] = nullptr;
        }
    }
};

struct sssp_graph {
    int device = 0;
    uint32_t n = 0;
    uint64_t m = 0;
    unsigned long long* d_off = nullptr;
    uint2* d_adj = nullptr;
    uint2* d_rows = nullptr;  // {row begin, degree} in 32 bits (m < 2^32): the throughput kernel's pop
    // locality relabeling (D15): internal id of each caller id (device, for finalize;
    // host, for the source); empty / nullptr = identity
    unsigned* d_perm = nullptr;
    std::vector<uint32_t> h_perm;
    uint32_t max_indeg = 0;
    uint64_t sum_w = 0;
    uint32_t max_w = 0;
    uint32_t heur_k_span = 0;  // log2 initial Delta, max_w / B rule (ring span)
    uint32_t heur_k_md = 0;    // log2 initial Delta, max_w / D rule
    uint32_t heur_k_nf = 0;    // log2 initial Delta, Near-Far C*W/D rule
    bool f32 = false;          // float32 weights (NEXT-3): max_w holds the IEEE bits
    sssp_options opts{};
    int sm_count = 0;
    std::vector<Workspace*> ws;
    DevBuf scratch, hostout, cert;
    cudaStream_t copy_stream = nullptr;  // device -> host copies of a host-output batch
    cudaEvent_t bev[2] = {nullptr, nullptr};  // batch start / end on the caller's stream
    int cur_bits = 32;       // 64 after a 32-bit overflow was observed (sticky)
    unsigned filt_shift_hint = 0;  // 1 + filter resolution fitted to the last run's max distance
    size_t persist_max = 0;  // device's L2 persisting set-aside limit (bytes)
    bool persist_saved = false;  // SSSP_FLAG_L2_PERSIST raised the device limit: restore after the run
    size_t persist_prev = 0;
    bool busy = false;
    bool async_pending = false;
    sssp_stats stats{};
};

namespace {

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

sssp_status check_options(const sssp_options& o) {
    if (o.struct_size != sizeof(sssp_options)) return fail(SSSP_ERR_INVALID_ARGUMENT, "options.struct_size mismatch");
    if (o.num_buckets < 2 || o.num_buckets > 32 || (o.num_buckets & (o.num_buckets - 1)))
        return fail(SSSP_ERR_INVALID_ARGUMENT, "num_buckets must be a power of two in [2, 32]");
    if (o.delta_mode > 1) return fail(SSSP_ERR_INVALID_ARGUMENT, "delta_mode");
    if (o.delta_heuristic > 2) return fail(SSSP_ERR_INVALID_ARGUMENT, "delta_heuristic");
    if (o.dist_bits != 0 && o.dist_bits != 32 && o.dist_bits != 64) return fail(SSSP_ERR_INVALID_ARGUMENT, "dist_bits");
    if (o.block_threads != 0 && o.block_threads != 128 && o.block_threads != 256 && o.block_threads != 512 &&
        o.block_threads != 1024)
        return fail(SSSP_ERR_INVALID_ARGUMENT, "block_threads must be 0, 128, 256, 512 or 1024");
    if (o.clip_pct == 0 || o.clip_pct > 100) return fail(SSSP_ERR_INVALID_ARGUMENT, "clip_pct");
    if (o.active_init > o.num_buckets) return fail(SSSP_ERR_INVALID_ARGUMENT, "active_init > num_buckets");
    if (o.waste_lo_permille > 1000 || o.waste_hi_permille > 1000) return fail(SSSP_ERR_INVALID_ARGUMENT, "waste permille");
    if (o.concurrent_sources > 64) return fail(SSSP_ERR_INVALID_ARGUMENT, "concurrent_sources > 64");
    if (o.algorithm > SSSP_ALGO_NEAR_FAR) return fail(SSSP_ERR_INVALID_ARGUMENT, "algorithm");
    if (o.worker > SSSP_WORKER_CTA)
        return fail(SSSP_ERR_INVALID_ARGUMENT, "worker: only SSSP_WORKER_AUTO / SSSP_WORKER_CTA (the warp-granular "
                                               "ablation was measured slower everywhere and removed, DESIGN.md D12)");
    return SSSP_OK;
}

// ----------------------------------------------------------------- kernel table
// Kernel variants: <dist type, CTA size, arcs per thread per round (EPT),
// arc-window size W>.  EPT = 4 independent L2 gathers in flight per thread;
// W = 2048 arcs (16 KB) prefetched asynchronously per window.
struct KVariant {
    void* fn;
    size_t smem;
};
template <typename DistT, int BT, bool kF = false, int EPT = 4, int MINB = 1024 / BT, bool PIPE = false, bool WLC = true,
          bool CA = false, int CHM = 2>
KVariant kvar() {
    // (without the warp-local loop the per-warp continuation queues are not allocated)
    return KVariant{(void*)adds_persistent_kernel<DistT, BT, EPT, MINB, PIPE, kF, WLC, CA, CHM>,
                    WLC ? Smem<DistT, BT, EPT>::bytes : Smem<DistT, BT, EPT>::o_wqv};
}
// The kernel instantiation for a launch shape (each variant's BT is the CTA size it
// is launched with).  32-bit distances: road-like graphs (warp-local build) run
// 128-thread CTAs x 4/SM at 128 registers (ROAD 40.8 -> 38.0 ms, sweeps §30) or
// 512 x 1/SM when asked; the throughput build is pipelined with claim-ahead at
// 512 x 2/SM (sweeps §8, §21).  64-bit distances and float32 weights use the plain
// build at the requested CTA size.
// The two default builds are compiled separately for flat (CHM 0) and chunked (CHM 1) bucket
// storage; every other instantiation decides at run time (CHM 2).
KVariant persistent_variant(int bits, int bt, bool f32, bool wlc, bool chunked, bool rows) {
    if (f32) return bt == 256 ? kvar<uint32_t, 256, true>() : kvar<uint32_t, 512, true>();
    if (bits == 32 && !wlc && !rows)  // (m >= 2^32: no 32-bit row records) the throughput build without them
        return kvar<uint32_t, 512, false, 4, 2, true, false, false>();
    if (bits == 32) {
        if (wlc && bt == 128)
            return chunked ? kvar<uint32_t, 128, false, 4, 4, true, true, false, 1>()
                           : kvar<uint32_t, 128, false, 4, 4, true, true, false, 0>();
        if (wlc && bt == 256) return kvar<uint32_t, 256, false, 4, 2, true>();
        if (wlc && bt == 512) return kvar<uint32_t, 512, false, 4, 1, true>();
        if (bt == 128) return kvar<uint32_t, 128, false, 4, 8, true, false, true>();
// (throughput build: 3 arcs per thread per round -- fewer live registers at the 64-register
// budget than 4: config 5 -3 %, ER -0.5 %; 2 is faster on config 5 but +1.5 % on ER, and 5-6
// spill: sweeps r02 §10)
#ifndef SSSP_TP_EPT
#define SSSP_TP_EPT 3
#endif
        if (bt == 512)
            return chunked ? kvar<uint32_t, 512, false, SSSP_TP_EPT, 2, true, false, true, 1>()
                           : kvar<uint32_t, 512, false, SSSP_TP_EPT, 2, true, false, true, 0>();
        if (bt == 1024) return kvar<uint32_t, 1024>();
        return kvar<uint32_t, 256, false, 4, 4, true, false, true>();  // throughput build, 4 CTAs/SM
    }
    if (bt == 128) return kvar<unsigned long long, 128>();
    if (bt == 512) return kvar<unsigned long long, 512>();
    if (bt == 1024) return kvar<unsigned long long, 1024>();
    return kvar<unsigned long long, 256>();
}

// warp-local continuation (D10): on for road-like graphs (average degree <= 8) unless disabled
bool warp_local_on(const sssp_graph* g) {
    if (g->opts.flags & (SSSP_FLAG_NO_LOCAL | SSSP_FLAG_NO_WARP_LOCAL)) return false;
    return (g->opts.flags & SSSP_FLAG_WARP_LOCAL) || g->m <= 8ull * g->n;
}

// Flat (default): items per bucket array, C >= n (no laps within a run, D13).  Chunked
// (SSSP_FLAG_CHUNKED_RING): items of the shared pool, 2n by default (bounded by the items alive
// at once, not by a run's pushes); ring_items overrides either.
bool chunked_ring(const sssp_graph* g) { return (g->opts.flags & SSSP_FLAG_CHUNKED_RING) != 0; }
unsigned long long default_cap(const sssp_graph* g) {
    if (g->opts.ring_items) return next_pow2(std::max<unsigned long long>(g->opts.ring_items, 64ull));
    if (chunked_ring(g)) return next_pow2(std::max<unsigned long long>(2ull * g->n, 1ull << 18));
    // road-like graphs (the latency build): 2n per slot -- at n = 2^24 ROAD overflowed 2^24-item
    // slots on some sources (the clip slot collects most of a run's far pushes), and each overflow
    // costs a full re-run (bench singles 31 -> 45 ms/source with two of them)
    const unsigned long long base = warp_local_on(g) ? 2ull * g->n : (unsigned long long)g->n;
    return next_pow2(std::max<unsigned long long>(base, 1ull << 16));
}

sssp_status ensure_ring(sssp_graph* g, Workspace& w, int item_bytes, unsigned long long cap) {
    const bool chunked = chunked_ring(g);
    unsigned pool_chunks = 0;
    if (chunked) {
        pool_chunks = (unsigned)std::min<unsigned long long>(
            next_pow2(std::max<unsigned long long>(cap >> kChunkShift, 64ull)), 1ull << 30);
        cap = (unsigned long long)pool_chunks << kChunkShift;
    }
    const size_t bytes = chunked ? (size_t)cap * item_bytes : (size_t)g->opts.num_buckets * cap * item_bytes;
    if (w.ring.p && w.ring.bytes >= bytes && w.cap == cap && w.ring_item_bytes == item_bytes && w.chunked == chunked)
        return SSSP_OK;
    w.ring.release();
    w.ctab.release();
    w.chunk_used.release();
    w.free_ring.release();
    w.pool.release();
    CK(cudaMalloc(&w.ring.p, bytes), "allocating the bucket ring");
    w.ring.bytes = bytes;
    CK(cudaMemset(w.ring.p, 0xFF, bytes), "clearing the bucket ring");
    if (chunked) {
        const size_t tb = (size_t)g->opts.num_buckets * pool_chunks * sizeof(unsigned);
        CK(cudaMalloc(&w.ctab.p, tb), "allocating the chunk tables");
        w.ctab.bytes = tb;
        CK(cudaMalloc(&w.chunk_used.p, (size_t)pool_chunks * 4), "allocating the chunk read counts");
        CK(cudaMalloc(&w.free_ring.p, (size_t)pool_chunks * 4), "allocating the free-chunk ring");
        CK(cudaMalloc(&w.pool.p, sizeof(ChunkPool)), "allocating the chunk pool counters");
    }
    w.chunked = chunked;
    w.pool_chunks = pool_chunks;
    w.cap = cap;
    w.ring_item_bytes = item_bytes;
    return SSSP_OK;
}

unsigned split_degree(const sssp_graph* g, unsigned bt) {
    if (g->opts.split_degree == 0xFFFFFFFFu) return 0u;
    // (chunk lengths must stay below the queue's slot-state markers, common.cuh)
    if (g->opts.split_degree) return std::min(g->opts.split_degree, 1u << 31);
    return 8u * bt;
}

// Hub-split chunk queue: enough entries for every arc of the graph in chunks of
// the smallest auto split degree (8 x 128), twice; doubled on overflow.
sssp_status ensure_tasks(sssp_graph* g, Workspace& w, unsigned long long tcap) {
    if (w.tasks.p && w.tcap == tcap) return SSSP_OK;
    w.tasks.release();
    const size_t bytes = (size_t)tcap * sizeof(SplitTask);
    CK(cudaMalloc(&w.tasks.p, bytes), "allocating the split-chunk queue");
    w.tasks.bytes = bytes;
    CK(cudaMemset(w.tasks.p, 0, bytes), "clearing the split-chunk queue");
    w.tcap = tcap;
    return SSSP_OK;
}
unsigned long long default_tcap(const sssp_graph* g) {
    return next_pow2(std::max<unsigned long long>(4096ull, 2ull * g->m / 1024ull));
}

sssp_status ensure_trace(sssp_graph* g, Workspace& w) {
    if (!(g->opts.flags & SSSP_FLAG_TRACE)) return SSSP_OK;
    unsigned cap = g->opts.trace_capacity ? g->opts.trace_capacity : 65536u;
    if (w.trace.p && w.trace_alloc >= cap) return SSSP_OK;
    w.trace.release();
    CK(cudaMalloc(&w.trace.p, (size_t)cap * sizeof(TraceEntry)), "allocating the trace ring");
    w.trace_alloc = cap;
    return SSSP_OK;
}

sssp_status alloc_workspace(sssp_graph* g, Workspace& w, bool own_stream) {
    const size_t n = g->n;
    CK(cudaMalloc(&w.dist.p, n * 8), "allocating dist");
    w.dist.bytes = n * 8;
    CK(cudaMalloc(&w.expanded.p, (n + 31) / 32 * 4), "allocating the expansion bitmap");
    CK(cudaMalloc(&w.filt.p, n * 2 + 16), "allocating the 16-bit filter");
    CK(cudaMalloc(&w.bk.p, sizeof(BucketCtl) * (kMaxBuckets + 1)), "allocating bucket counters");
    CK(cudaMemset(w.bk.p, 0, sizeof(BucketCtl) * (kMaxBuckets + 1)), "bucket counters");
    CK(cudaMalloc(&w.ctl.p, sizeof(Ctl)), "allocating control block");
    CK(cudaMemset(w.ctl.p, 0, sizeof(Ctl)), "control block");
    CK(cudaHostAlloc((void**)&w.h_ctl, sizeof(Ctl), cudaHostAllocMapped), "allocating pinned status block");
    CK(cudaHostGetDevicePointer((void**)&w.h_ctl_dev, w.h_ctl, 0), "mapping the status block");
    std::memset(w.h_ctl, 0, sizeof(Ctl));
    for (auto& e : w.ev) CK(cudaEventCreate(&e), "creating events");
    if (own_stream) CK(cudaStreamCreateWithFlags(&w.own_stream, cudaStreamNonBlocking), "creating a slot stream");
    sssp_status st = ensure_tasks(g, w, default_tcap(g));
    if (st) return st;
    return ensure_ring(g, w, (g->opts.dist_bits == 64) ? 16 : 8, default_cap(g));
}

sssp_status ensure_slots(sssp_graph* g, unsigned c) {
    while (g->ws.size() < c) {
        Workspace* w = new Workspace();
        g->ws.push_back(w);
        sssp_status st = alloc_workspace(g, *w, g->ws.size() > 1);
        if (st) {
            w->release();
            delete w;
            g->ws.pop_back();
            return st;
        }
    }
    return SSSP_OK;
}

template <typename DistT>
Params<DistT> make_params(sssp_graph* g, Workspace& w, unsigned grid, unsigned bt, unsigned k_max, unsigned conc) {
    Params<DistT> p{};
    p.off = g->d_off;
    p.adj = g->d_adj;
    p.rows = (g->opts.flags & SSSP_FLAG_WIDE_ROWS) ? nullptr : g->d_rows;
    p.dist = (DistT*)w.dist.p;
    p.ring = (char*)w.ring.p;
    p.chunked = w.chunked ? 1u : 0u;
    p.ctab = (unsigned*)w.ctab.p;
    p.tab_mask = w.pool_chunks ? w.pool_chunks - 1 : 0u;
    p.chunk_used = (unsigned*)w.chunk_used.p;
    p.free_ring = (unsigned*)w.free_ring.p;
    p.pool = (ChunkPool*)w.pool.p;
    p.pool_chunks = w.pool_chunks;
    p.bk = (BucketCtl*)w.bk.p;
    p.ctl = (Ctl*)w.ctl.p;
    const bool tr = (g->opts.flags & SSSP_FLAG_TRACE) != 0;
    p.trace = tr ? (TraceEntry*)w.trace.p : nullptr;
    p.trace_cap = tr ? w.trace_alloc : 0;
    p.n = g->n;
    p.nb = g->opts.num_buckets;
    p.cap = w.cap;
    p.dynamic = g->opts.delta_mode == SSSP_DELTA_DYNAMIC;
    // active buckets adapt by default; SSSP_FLAG_FIXED_ACTIVE pins them at active_init
    p.adapt_active = (g->opts.flags & SSSP_FLAG_FIXED_ACTIVE) ? 0u : 1u;
    p.grid = grid;
    p.clip_pct = g->opts.clip_pct;
    p.settle = g->opts.settle_head_switches;
    p.util_lo_pct = g->opts.util_lo_pct;
    p.util_hi_pct = g->opts.util_hi_pct;
    p.resident_threads = (unsigned long long)grid * bt;
    const double deg = g->n ? (double)g->m / g->n : 0.0;
    p.avg_deg_x16 = (unsigned)std::min(16.0 * deg + 0.5, 4.0e9);
    // auto: 256 on the throughput side (fewer, larger batches: RMAT/ER -1.7 %, sweeps r02 §10),
    // 32 on road-like graphs (large batches there break the latency regime: ROAD work 70x)
    p.batch_min = g->opts.batch_min ? g->opts.batch_min : (warp_local_on(g) ? 32u : 256u);
    unsigned sh = 0;
    while ((1u << (sh + 1)) <= grid) ++sh;  // floor(log2 grid)
    p.share_shift = sh > 2 ? sh - 2 : 0;
    p.local_max = (g->opts.flags & SSSP_FLAG_NO_LOCAL) ? 0u : (g->opts.local_max ? g->opts.local_max : 128u);
    // warp-local continuation pays on low-degree graphs (road-like: each lane's row fits
    // one or two rounds of EPT arcs); on ER (degree 32) it serialised what the ring spreads
    // over CTAs (measured +13 %), so it is on by default only for average degree <= 8
    p.warp_local = warp_local_on(g) ? 1u : 0u;
    p.max_backoff_ns = g->opts.max_backoff_ns ? g->opts.max_backoff_ns : (p.warp_local ? 512u : 2048u);  // §30
    p.prof = (g->opts.flags & SSSP_FLAG_PROFILE) ? 1u : 0u;
    p.expanded = (unsigned*)w.expanded.p;
    p.waste_lo = g->opts.waste_lo_permille;
    p.waste_hi = g->opts.waste_hi_permille;
    p.startup_first = (unsigned long long)g->n * g->opts.startup_permille / 1000ull;
    p.period_ns = (unsigned long long)(g->opts.period_us ? g->opts.period_us : 20u) * 1000ull;
    // L2 residency of dist (D5): reserve the persisting set-aside for
    // the concurrently live dist arrays and mark dist accesses evict_last over
    // the fraction that fits
    // The device-wide set-aside is touched only when the caller opts in; the previous
    // limit is restored when the run ends (restore_persist).
    p.keep_frac = 0.0f;
    if ((g->opts.flags & SSSP_FLAG_L2_PERSIST) && g->persist_max) {
        const size_t want = (size_t)g->n * sizeof(DistT) * conc;
        const size_t use = std::min(want, g->persist_max);
        size_t cur = 0;
        cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
        if (!g->persist_saved) {
            g->persist_saved = true;
            g->persist_prev = cur;
        }
        if (cur < use) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, use);
        cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
        p.keep_frac = want ? (float)std::min(1.0, (double)std::min(cur, use) / (double)want) : 0.0f;
    }
    // 16-bit filter (D11, opt-in): integer weights only (distances beyond
    // 65534 * 2^s simply have no bound and go to the atomic)
    {
        const bool on = !g->f32 && (g->opts.flags & SSSP_FLAG_FILTER16);
        unsigned lg = 0;
        while (lg < 31 && (2u << lg) <= g->max_w) ++lg;  // floor(log2 max_w)
        p.filt = on ? (unsigned short*)w.filt.p : nullptr;
        // first run on a graph: 2^s = max_w / 16; afterwards the resolution that maps the
        // previous run's largest distance below 60000 (the result never depends on it)
        p.filt_shift = g->filt_shift_hint ? g->filt_shift_hint - 1 : (lg > 4 ? lg - 4 : 0);
    }
    p.tasks = (SplitTask*)w.tasks.p;
    p.tcap = w.tcap;
    p.split_deg = split_degree(g, bt);
    p.k_max = k_max;
    p.timeout_ns = (unsigned long long)(g->opts.timeout_ms ? g->opts.timeout_ms : 60000u) * 1000000ull;
    return p;
}

unsigned heuristic_k(const sssp_graph* g) {
    if (g->f32) {  // Delta = 2^(k - kFloatBias): ring span max_w / B in float
        union {
            unsigned u;
            float f;
        } mw{g->max_w};
        const double q = (double)mw.f / (double)g->opts.num_buckets;
        const long e = q > 0 ? std::lround(std::log2(q)) : -40;
        return (unsigned)std::min<long>(std::max<long>(e + kFloatBias, 0), 190);
    }
    switch (g->opts.delta_heuristic) {
        case SSSP_DELTA_H_NEARFAR: return g->heur_k_nf;
        case SSSP_DELTA_H_MAXW_OVER_D: return g->heur_k_md;
        default: return std::min(ilog2_round((double)g->max_w / (double)g->opts.num_buckets), 63u);
    }
}

// One attempt of one source with `bits`-wide internal distances on workspace w.
// `conc` workspaces share the GPU: each persistent grid gets 1/conc of the CTAs.
// (The kernel never waits on a CTA that has not started -- no grid barrier --
// so co-residency is not required; one slot launches cooperatively anyway.)
template <typename DistT, bool kF>
sssp_status launch_one(sssp_graph* g, Workspace& w, uint32_t source, void* out_dev, cudaStream_t s, int bits,
                       unsigned k0, unsigned conc) {
    // auto CTA size: 512, except road-like graphs (warp-local build, 32-bit distances): four
    // 128-thread CTAs per SM at the same 128-register budget -- more independent claimers on a
    // latency-bound graph (ROAD 40.8 -> 38.0 ms with the 512 ns backoff cap, sweeps §30)
    const bool wlc_auto = !kF && bits == 32 && warp_local_on(g);
    unsigned bt = g->opts.block_threads ? g->opts.block_threads : (wlc_auto ? 128u : 512u);
    if (kF && bt != 256) bt = 512;  // float variants are built for 256/512-thread CTAs
    const bool rows32 = g->d_rows && !(g->opts.flags & SSSP_FLAG_WIDE_ROWS);
    if (!kF && bits == 32 && !warp_local_on(g) && !rows32) bt = 512;  // (see persistent_variant)
    const KVariant kv = persistent_variant(bits, (int)bt, kF, warp_local_on(g), chunked_ring(g), rows32);
    void* fn = kv.fn;
    CK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kv.smem), "smem attribute");
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, (int)bt, kv.smem), "occupancy query");
    if (occ < 1) return fail(SSSP_ERR_CUDA, "persistent kernel cannot be resident");
    unsigned grid = (unsigned)(occ * g->sm_count);
    if (g->opts.grid_ctas && g->opts.grid_ctas < grid) grid = g->opts.grid_ctas;
    grid = std::max(1u, grid / conc);
    const unsigned k_max = kF ? 190u : (bits == 32 ? 31u : 63u);
    unsigned k = std::min(k0, k_max);
    // active buckets: auto = 4 on the throughput build (average degree > 8) -- CTAs
    // that find the head bucket's published items exhausted take the next buckets' instead of
    // idling through the head's tail (vs 1: RMAT -20 %, ER -17 %; vs 2: -1..4 %, sweeps §26) --
    // and 1 on road-like graphs, where 2 gained only 2 % with more run-to-run spread and 3 sent
    // the controller into a shrink spiral
    const unsigned A0 = g->opts.active_init ? g->opts.active_init : (g->m > 8ull * g->n ? 4u : 1u);
    // initial floor of Delta (the controller never shrinks below it; clipping raises it):
    // 8x below the ring-span value w_max / B (below which one maximum-weight hop from the head
    // lands beyond the ring).  Graphs whose distances are made of small weights need the
    // room: RMAT with U[1,2^20] has its best static Delta at or below 2^13 with the span at 2^15
    // (reading R8, profiles/r02_sweeps.md §7)
    const unsigned span = kF ? heuristic_k(g) : g->heur_k_span;
    Head h0{0ull, pack_meta(0, k, A0, std::min(k, span > 3 ? span - 3 : 0u), 0)};
    Params<DistT> p = make_params<DistT>(g, w, grid, bt, k_max, conc);
    p.a_min = A0;
    p.a_max = std::min(g->opts.num_buckets, std::max(2u, 2u * A0));

    const unsigned aux_grid = (unsigned)g->sm_count * 8 / conc + 1;
    CK(cudaEventRecord(w.ev[0], s), "event");
    if (!g->h_perm.empty()) source = g->h_perm[source];  // internal id (D15)
    ChunkInit cinit;
    if (p.chunked) {
        cinit.ctab = p.ctab;
        cinit.tab_stride = p.tab_mask + 1;
        cinit.nb = p.nb;
        cinit.chunk_used = p.chunk_used;
        cinit.free_ring = p.free_ring;
        cinit.pool_chunks = p.pool_chunks;
        cinit.pool = p.pool;
    }
    init_run_kernel<DistT><<<aux_grid, 256, 0, s>>>(p.dist, g->n, source, p.ctl, p.bk, p.ring, w.cap, h0,
                                                    p.expanded, p.filt, cinit);
    CK(cudaGetLastError(), "init kernel launch");
    CK(cudaEventRecord(w.ev[1], s), "event");
    void* args[] = {(void*)&p};
    if (conc == 1) {
        CK(cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(bt), args, kv.smem, s), "persistent kernel launch");
    } else {
        CK(cudaLaunchKernel(fn, dim3(grid), dim3(bt), args, kv.smem, s), "persistent kernel launch");
    }
    CK(cudaEventRecord(w.ev[2], s), "event");
    if constexpr (kF)
        finalize_f32_kernel<<<aux_grid, 256, 0, s>>>((const unsigned*)p.dist, (float*)out_dev, g->n, g->d_off, p.ctl,
                                                     g->d_perm);
    else
        finalize_kernel<DistT><<<aux_grid, 256, 0, s>>>(p.dist, (unsigned long long*)out_dev, g->n, g->d_off, p.ctl,
                                                        g->d_perm);
    CK(cudaGetLastError(), "finalize kernel launch");
    CK(cudaEventRecord(w.ev[3], s), "event");
    status_copy_kernel<<<1, 256, 0, s>>>((const unsigned long long*)w.ctl.p, (unsigned long long*)w.h_ctl_dev,
                                         (unsigned)(sizeof(Ctl) / 8));
    CK(cudaGetLastError(), "status copy");
    w.last_grid = grid;
    w.last_block = bt;
    w.last_worker = SSSP_WORKER_CTA;
    w.last_k0 = k;
    return SSSP_OK;
}

// ------------------------------------------------------------ Near-Far ablation (NEXT-2)
sssp_status ensure_nf(sssp_graph* g, Workspace& w, int item_bytes, unsigned long long cap) {
    if (w.nf_piles.p && w.nf_cap == cap && w.nf_item_bytes == item_bytes) return SSSP_OK;
    w.nf_piles.release();
    CK(cudaMalloc(&w.nf_piles.p, 4 * (size_t)cap * item_bytes), "allocating Near-Far piles");
    w.nf_piles.bytes = 4 * (size_t)cap * item_bytes;
    if (!w.nf_cnt.p) CK(cudaMalloc(&w.nf_cnt.p, sizeof(NFCounters)), "allocating Near-Far counters");
    w.nf_cap = cap;
    w.nf_item_bytes = item_bytes;
    return SSSP_OK;
}

template <typename DistT>
sssp_status launch_nf(sssp_graph* g, Workspace& w, uint32_t source, void* out_dev_v, cudaStream_t s,
                      int bits, unsigned k0) {
    unsigned long long* out_dev = (unsigned long long*)out_dev_v;
    const int ib = bits == 32 ? 8 : 16;
    sssp_status st = ensure_nf(g, w, ib, w.nf_cap ? w.nf_cap : 2 * default_cap(g));
    if (st) return st;
    void* fn = (void*)near_far_kernel<DistT>;
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, 256, 0), "occupancy query");
    unsigned grid = (unsigned)(std::max(occ, 1) * g->sm_count);
    if (g->opts.grid_ctas && g->opts.grid_ctas < grid) grid = g->opts.grid_ctas;
    NFParams<DistT> p{};
    p.off = g->d_off;
    p.adj = g->d_adj;
    p.dist = (DistT*)w.dist.p;
    unsigned long long* base = (unsigned long long*)w.nf_piles.p;
    const size_t words = (size_t)w.nf_cap * (ib / 8);
    p.near[0] = base;
    p.near[1] = base + words;
    p.far[0] = base + 2 * words;
    p.far[1] = base + 3 * words;
    p.cnt = (NFCounters*)w.nf_cnt.p;
    p.ctl = (Ctl*)w.ctl.p;
    p.cap = w.nf_cap;
    p.delta = 1ull << std::min(k0, bits == 32 ? 31u : 62u);
    p.timeout_ns = (unsigned long long)(g->opts.timeout_ms ? g->opts.timeout_ms : 60000u) * 1000000ull;
    const unsigned aux_grid = (unsigned)g->sm_count * 8;
    CK(cudaEventRecord(w.ev[0], s), "event");
    if (!g->h_perm.empty()) source = g->h_perm[source];  // internal id (D15)
    near_far_init_kernel<DistT><<<aux_grid, 256, 0, s>>>(p.dist, g->n, source, p.cnt, p.ctl, p.near[0]);
    CK(cudaGetLastError(), "init kernel launch");
    CK(cudaEventRecord(w.ev[1], s), "event");
    void* args[] = {(void*)&p};
    CK(cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(256), args, 0, s), "Near-Far kernel launch");
    CK(cudaEventRecord(w.ev[2], s), "event");
    finalize_kernel<DistT><<<aux_grid, 256, 0, s>>>(p.dist, out_dev, g->n, g->d_off, p.ctl, g->d_perm);
    CK(cudaGetLastError(), "finalize kernel launch");
    CK(cudaEventRecord(w.ev[3], s), "event");
    status_copy_kernel<<<1, 256, 0, s>>>((const unsigned long long*)w.ctl.p, (unsigned long long*)w.h_ctl_dev,
                                         (unsigned)(sizeof(Ctl) / 8));
    CK(cudaGetLastError(), "status copy");
    w.last_grid = grid;
    w.last_block = 256;
    w.last_worker = 0;
    w.last_k0 = std::min(k0, bits == 32 ? 31u : 62u);
    return SSSP_OK;
}

sssp_status launch_attempt(sssp_graph* g, Workspace& w, uint32_t source, void* out_dev, cudaStream_t s,
                           int bits, unsigned conc) {
    if (g->f32) {
        if (g->opts.algorithm == SSSP_ALGO_NEAR_FAR)
            return fail(SSSP_ERR_INVALID_ARGUMENT, "the Near-Far ablation supports integer weights only");
        const unsigned k0 = g->opts.delta_init ? kFloatBias + ilog2_round((double)g->opts.delta_init) : heuristic_k(g);
        sssp_status st = ensure_ring(g, w, 8, w.cap ? w.cap : default_cap(g));
        if (st) return st;
        if ((st = ensure_trace(g, w))) return st;
        return launch_one<uint32_t, true>(g, w, source, out_dev, s, 32, k0, conc);
    }
    if (g->opts.algorithm == SSSP_ALGO_NEAR_FAR) {
        // static Delta: the Near-Far rule unless given
        const unsigned k0 = g->opts.delta_init ? ilog2_round((double)g->opts.delta_init) : g->heur_k_nf;
        if (bits == 32) return launch_nf<uint32_t>(g, w, source, out_dev, s, 32, k0);
        return launch_nf<unsigned long long>(g, w, source, out_dev, s, 64, k0);
    }
    const unsigned k0 = g->opts.delta_init ? ilog2_round((double)g->opts.delta_init) : heuristic_k(g);
    sssp_status st = ensure_ring(g, w, bits == 32 ? 8 : 16, w.cap ? w.cap : default_cap(g));
    if (st) return st;
    if ((st = ensure_trace(g, w))) return st;
    if (bits == 32) return launch_one<uint32_t, false>(g, w, source, out_dev, s, 32, k0, conc);
    return launch_one<unsigned long long, false>(g, w, source, out_dev, s, 64, k0, conc);
}

void accumulate(sssp_graph* g, Workspace& w, const Ctl& c, int bits) {
    sssp_stats& st = g->stats;
    st.vertices_processed += c.st_vertices;
    st.edges_relaxed += c.st_edges;
    st.pushes += c.st_pushes + 1;  // + the source item
    st.stale_skips += c.st_stale;
    st.reachable += c.reach_v;
    st.reach_edges += c.reach_e;
    st.max_dist = std::max<uint64_t>(st.max_dist, c.max_dist);
    if (!g->f32 && c.max_dist) {  // resolution of the 16-bit filter for the next run on this graph
        unsigned sh = 0;
        while (sh < 48 && (c.max_dist >> sh) >= 60000ull) ++sh;
        g->filt_shift_hint = sh + 1;  // stored +1 (0 = no run yet)
    }
    st.init_delta_log2 = w.last_k0;
    st.final_delta_log2 = g->opts.algorithm == SSSP_ALGO_NEAR_FAR ? w.last_k0 : meta_k(c.head.meta);
    st.head_switches += c.head_switches;
    st.delta_changes += c.delta_changes;
    st.dist_bits = (uint32_t)bits;
    st.grid_ctas = w.last_grid;
    st.block_threads = w.last_block;
    st.worker = w.last_worker;
    st.ring_bytes = std::max<uint64_t>(st.ring_bytes, w.ring.bytes + w.ctab.bytes + 8ull * w.pool_chunks);
    st.runs += 1;
    st.trace_entries = std::min<uint32_t>(c.trace_count, w.trace_alloc);
    float a = 0, b = 0;
    cudaEventElapsedTime(&a, w.ev[1], w.ev[2]);
    cudaEventElapsedTime(&b, w.ev[0], w.ev[3]);
    st.kernel_ms += a;
    st.total_ms += b;
}

// An aborted attempt leaves items in the bucket ring and chunks in the hub-split
// queue (init_run_kernel resets only the counters): wipe both before the
// workspace is used again (shared by the synchronous retry path and the
// SSSP_FLAG_ASYNC error path of sssp_get_stats).
sssp_status clear_after_abort(Workspace& w, cudaStream_t s) {
    CK(cudaMemsetAsync(w.ring.p, 0xFF, w.ring.bytes, s), "clearing the bucket ring");
    if (w.tasks.p) CK(cudaMemsetAsync(w.tasks.p, 0, w.tasks.bytes, s), "clearing the split-chunk queue");
    CK(cudaStreamSynchronize(s), "clearing the bucket ring");
    return SSSP_OK;
}

// Inspect a finished attempt.  Returns SSSP_OK and sets *done on success; on a
// recoverable device status prepares the retry (clears/grows the ring, switches
// to 64-bit) and leaves *done false; otherwise returns the error.
sssp_status settle_attempt(sssp_graph* g, Workspace& w, cudaStream_t s, int& bits, int attempt, bool* done) {
    *done = false;
    const unsigned status = w.h_ctl->status;
    if (status == 0) {
        accumulate(g, w, *w.h_ctl, bits);
        *done = true;
        return SSSP_OK;
    }
    sssp_status cst = clear_after_abort(w, s);
    if (cst) return cst;
    if (status & kStTimeout) return fail(SSSP_ERR_TIMEOUT, "device watchdog expired");
    if (status & kStBug) return fail(SSSP_ERR_CUDA, "internal invariant violated");
    if (status & kStDistOverflow) {
        if (g->opts.dist_bits == 32) return fail(SSSP_ERR_INVALID_ARGUMENT, "distances exceed 32 bits (dist_bits=32)");
        bits = 64;
        if (!g->opts.dist_bits) g->cur_bits = 64;
        g->stats.retries += 1;
        return SSSP_OK;
    }
    if (status & kStRingOverflow) {
        if ((g->opts.flags & SSSP_FLAG_NO_RETRY) || attempt >= 20)
            return fail(SSSP_ERR_WORKLIST_OVERFLOW, "bucket ring overflow");
        if (g->opts.algorithm == SSSP_ALGO_NEAR_FAR) {
            sssp_status st2 = ensure_nf(g, w, w.nf_item_bytes, w.nf_cap * 2);
            if (st2) return st2;
            g->stats.retries += 1;
            return SSSP_OK;
        }
        const unsigned long long ncap = w.cap * 2;
        sssp_status st3 = ensure_tasks(g, w, w.tcap * 2);
        if (st3) return st3;
        w.ring.release();
        sssp_status st2 = ensure_ring(g, w, bits == 32 ? 8 : 16, ncap);
        if (st2) return st2;
        g->stats.retries += 1;
        return SSSP_OK;
    }
    return fail(SSSP_ERR_CUDA, "unknown device status");
}

// Synchronous run of one source on one workspace, with retry.
sssp_status run_one_sync(sssp_graph* g, Workspace& w, uint32_t source, void* out_dev, cudaStream_t s,
                         unsigned conc) {
    int bits = g->opts.dist_bits ? (int)g->opts.dist_bits : g->cur_bits;
    for (int attempt = 0; attempt < 24; ++attempt) {
        sssp_status st = launch_attempt(g, w, source, out_dev, s, bits, conc);
        if (st) return st;
        CK(cudaStreamSynchronize(s), "SSSP run");
        bool done = false;
        if ((st = settle_attempt(g, w, s, bits, attempt, &done))) return st;
        if (done) return SSSP_OK;
    }
    return fail(SSSP_ERR_WORKLIST_OVERFLOW, "retries exhausted");
}

sssp_status classify_out(sssp_graph* g, const void* ptr, bool* is_dev) {
    cudaPointerAttributes a{};
    cudaError_t e = cudaPointerGetAttributes(&a, ptr);
    if (e != cudaSuccess) {
        cudaGetLastError();
        *is_dev = false;
        return SSSP_OK;
    }
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) {
        if (a.device != g->device) return fail(SSSP_ERR_DEVICE_MISMATCH, "dist_out is on another device");
        *is_dev = true;
    } else {
        *is_dev = false;
    }
    return SSSP_OK;
}

// Concurrent batch (device dist_out): groups of c sources, one per workspace
// and stream; every attempt of a group is launched before any is awaited.
// c sources in flight, one per workspace slot.  Host dist_out (`host`): each slot finalizes into
// one of its two device staging rows and the row goes to the host on the graph's copy stream
// while the next sources compute (the copy of group i overlaps groups i+1 and i+2; a staging row
// is rewritten only after its copy's event).
sssp_status run_concurrent(sssp_graph* g, const uint32_t* sources, uint32_t k, char* out, size_t esz,
                           cudaStream_t caller, unsigned c, bool host = false) {
    sssp_status st = ensure_slots(g, c);
    if (st) return st;
    if (host) {
        if (!g->copy_stream) CK(cudaStreamCreateWithFlags(&g->copy_stream, cudaStreamNonBlocking), "copy stream");
        for (unsigned j = 0; j < c; ++j)
            for (int b = 0; b < 2; ++b) {
                Workspace& w = *g->ws[j];
                if (!w.stage[b].p) {
                    CK(cudaMalloc(&w.stage[b].p, (size_t)g->n * 8), "allocating a staging row");
                    w.stage[b].bytes = (size_t)g->n * 8;
                }
                if (!w.cev[b]) CK(cudaEventCreateWithFlags(&w.cev[b], cudaEventDisableTiming), "event");
                CK(cudaEventRecord(w.cev[b], g->copy_stream), "event");
            }
    }
    CK(cudaEventRecord(g->bev[0], caller), "event");
    for (unsigned j = 1; j < c; ++j) CK(cudaStreamWaitEvent(g->ws[j]->own_stream, g->bev[0], 0), "stream join");
    auto slot_stream = [&](unsigned j) { return j == 0 ? caller : g->ws[j]->own_stream; };
    // Every slot runs its own sequence: when a slot's source finishes (stream query), it is
    // settled and the slot starts the next source at once -- no slot waits for the slowest
    // source of a group.
    constexpr uint32_t kNone = 0xFFFFFFFFu;
    std::vector<uint32_t> run_i(c, kNone);  // source index running in slot j
    std::vector<int> run_bits(c, 32);
    std::vector<unsigned> spar(c, 1u);      // slot j's staging row (host output)
    std::vector<int> tries(c, 0);           // attempts of the running source (overflow re-runs)
    uint32_t next = 0;
    unsigned active = 0;
    auto out_of = [&](unsigned j, uint32_t i) -> void* {
        return host ? g->ws[j]->stage[spar[j]].p : (void*)(out + (size_t)i * g->n * esz);
    };
    auto start = [&](unsigned j) -> sssp_status {
        const uint32_t i = next++;
        if (host) {  // the staging row's previous copy (two sources back on this slot) has left it
            spar[j] ^= 1u;
            CK(cudaStreamWaitEvent(slot_stream(j), g->ws[j]->cev[spar[j]], 0), "stream wait");
        }
        run_i[j] = i;
        run_bits[j] = g->opts.dist_bits ? (int)g->opts.dist_bits : g->cur_bits;
        tries[j] = 0;
        ++active;
        return launch_attempt(g, *g->ws[j], sources[i], out_of(j, i), slot_stream(j), run_bits[j], c);
    };
    for (unsigned j = 0; j < c && next < k && st == SSSP_OK; ++j) st = start(j);
    while (active && st == SSSP_OK) {
        bool any = false;
        for (unsigned j = 0; j < c && st == SSSP_OK; ++j) {
            if (run_i[j] == kNone) continue;
            const cudaError_t q = cudaStreamQuery(slot_stream(j));
            if (q == cudaErrorNotReady) continue;
            if (q != cudaSuccess) {
                st = cuda_fail(q, "SSSP run");
                break;
            }
            any = true;
            const uint32_t i = run_i[j];
            int b = run_bits[j];
            bool done = false;
            st = settle_attempt(g, *g->ws[j], slot_stream(j), b, tries[j], &done);
            if (st == SSSP_OK && !done) {  // recoverable (ring regrown / 64-bit): re-run it on this slot,
                run_bits[j] = b;             // without holding up the other slots
                if (++tries[j] >= 24) st = fail(SSSP_ERR_WORKLIST_OVERFLOW, "retries exhausted");
                else st = launch_attempt(g, *g->ws[j], sources[i], out_of(j, i), slot_stream(j), b, c);
                continue;
            }
            if (st == SSSP_OK && host) {  // the row is final: send it home on the copy stream
                cudaError_t e = cudaMemcpyAsync(out + (size_t)i * g->n * esz, g->ws[j]->stage[spar[j]].p,
                                                (size_t)g->n * esz, cudaMemcpyDeviceToHost, g->copy_stream);
                if (e == cudaSuccess) e = cudaEventRecord(g->ws[j]->cev[spar[j]], g->copy_stream);
                if (e != cudaSuccess) st = cuda_fail(e, "copying dist to host");
            }
            run_i[j] = kNone;
            --active;
            if (st == SSSP_OK && next < k) st = start(j);
        }
        if (!any && st == SSSP_OK) std::this_thread::sleep_for(std::chrono::microseconds(5));
    }
    if (st != SSSP_OK)  // drain the slots still running before the workspaces are reused
        for (unsigned j = 0; j < c; ++j)
            if (run_i[j] != kNone) cudaStreamSynchronize(slot_stream(j));
    for (unsigned j = 1; j < c; ++j) {
        cudaEventRecord(g->ws[j]->ev[3], g->ws[j]->own_stream);
        cudaStreamWaitEvent(caller, g->ws[j]->ev[3], 0);
    }
    if (host) {
        const cudaError_t e = cudaStreamSynchronize(g->copy_stream);  // host rows complete on return
        if (e != cudaSuccess && st == SSSP_OK) st = cuda_fail(e, "copying dist to host");
    }
    return st;
}

void restore_persist(sssp_graph* g) {
    if (!g->persist_saved) return;
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, g->persist_prev);
    g->persist_saved = false;
}

sssp_status run_many(sssp_graph* g, const uint32_t* sources, uint32_t k, void* dist_out, bool f32_out,
                     sssp_stream_t stream) {
    if (!g || !dist_out || (k && !sources)) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL argument");
    if (f32_out != g->f32)
        return fail(SSSP_ERR_INVALID_ARGUMENT, g->f32 ? "float32-weight graph: use sssp_run_f32 / sssp_run_batch_f32"
                                                      : "integer-weight graph: use sssp_run / sssp_run_batch");
    const size_t esz = g->f32 ? 4 : 8;
    if (k == 0) return fail(SSSP_ERR_INVALID_ARGUMENT, "k == 0");
    for (uint32_t i = 0; i < k; ++i)
        if (sources[i] >= g->n) return fail(SSSP_ERR_INVALID_ARGUMENT, "source " + std::to_string(sources[i]) + " >= n");
    if (g->busy || g->async_pending) return fail(SSSP_ERR_BUSY, "a run is already in flight on this handle");
    DeviceGuard dg(g->device);
    bool is_dev = false;
    sssp_status st = classify_out(g, dist_out, &is_dev);
    if (st) return st;
    cudaStream_t s = (cudaStream_t)stream;
    g->busy = true;
    g->stats = sssp_stats{};
    Workspace& w0 = *g->ws[0];
    const unsigned c = g->opts.algorithm == SSSP_ALGO_NEAR_FAR
                           ? 1u  // grid-wide barriers: one cooperative launch at a time
                           : std::min<unsigned>(std::max(1u, g->opts.concurrent_sources), k);
    g->stats.concurrency = c > 1 ? c : 1;
    const bool async = (g->opts.flags & SSSP_FLAG_ASYNC) && is_dev && k == 1;
    if (!is_dev && !g->hostout.p) {
        cudaError_t e = cudaMalloc(&g->hostout.p, (size_t)g->n * 8);
        if (e != cudaSuccess) {
            g->busy = false;
            return cuda_fail(e, "allocating the staging buffer for a host dist_out");
        }
        g->hostout.bytes = (size_t)g->n * 8;
    }
    cudaEventRecord(g->bev[0], s);
    if (c > 1) {  // (host dist_out: staged per slot, copies overlapped with the next sources)
        st = run_concurrent(g, sources, k, (char*)dist_out, esz, s, c, !is_dev);
    } else {
        for (uint32_t i = 0; i < k && st == SSSP_OK; ++i) {
            void* out = is_dev ? (void*)((char*)dist_out + (size_t)i * g->n * esz) : g->hostout.p;
            if (async) {
                const int bits = g->opts.dist_bits ? (int)g->opts.dist_bits : g->cur_bits;
                st = launch_attempt(g, w0, sources[i], out, s, bits, 1);
                if (st == SSSP_OK) {
                    g->async_pending = true;
                    g->stats.dist_bits = (uint32_t)bits;
                }
            } else {
                st = run_one_sync(g, w0, sources[i], out, s, 1);
                if (st == SSSP_OK && !is_dev) {
                    cudaError_t e = cudaMemcpyAsync((char*)dist_out + (size_t)i * g->n * esz, out, (size_t)g->n * esz,
                                                    cudaMemcpyDeviceToHost, s);
                    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
                    if (e != cudaSuccess) st = cuda_fail(e, "copying dist to host");
                }
            }
        }
    }
    cudaEventRecord(g->bev[1], s);
    if (!async && st == SSSP_OK) {
        cudaEventSynchronize(g->bev[1]);
        float ms = 0;
        cudaEventElapsedTime(&ms, g->bev[0], g->bev[1]);
        g->stats.batch_ms = ms;
    }
    if (!async) restore_persist(g);
    g->stats.status = st;
    g->busy = false;
    return st;
}

}  // namespace

// =================================================================== C ABI
extern "C" {

void sssp_options_default(sssp_options* o) {
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->struct_size = sizeof(sssp_options);
    o->device = 0;
    o->num_buckets = 32;
    o->delta_mode = SSSP_DELTA_DYNAMIC;
    o->delta_init = 0;             // 0 = heuristic (delta_heuristic; default ring span w_max/B, reading R3)
    o->clip_pct = 65;
    o->settle_head_switches = 8;   // P:215 (reading R7): controller steps between Delta changes
    o->util_lo_pct = 100;          // P:211 (reading R6)
    o->util_hi_pct = 400;
    o->waste_lo_permille = 500;    // reading R6: grow Delta only while < 50% of expansions are repeats
    o->waste_hi_permille = 600;    //             shrink it while > 60% are (work <~ 2.5x Dijkstra)
    o->period_us = 20;
    o->startup_permille = 20;
    o->dist_bits = 0;
    o->ring_items = 0;
    o->flags = 0;
    o->block_threads = 0;
    o->grid_ctas = 0;
    o->batch_min = 0;
    o->timeout_ms = 0;
    o->trace_capacity = 0;
    o->active_init = 0;
    o->concurrent_sources = 1;
}

}  // extern "C"

namespace {
// Locality relabeling (D15): renumber vertices by descending in-degree so
// the dist entries that most arcs gather from and atomically update share cache
// lines (on a power-law graph the hot set becomes a few MB of L2-resident lines
// instead of one hot entry per 32-byte sector).  The distance vector is a property
// of the graph, not of its numbering: the source is mapped in, finalize gathers the
// output back in caller order, so results are bit-identical.  Auto: on when the
// in-degree is skewed (max > 64 x average); SSSP_FLAG_RELABEL / SSSP_FLAG_NO_RELABEL
// force it.
sssp_status relabel_graph(sssp_graph* g, const sssp_options& o) {
    const unsigned n = g->n;
    const unsigned long long m = g->m;
    const unsigned aux_grid = (unsigned)g->sm_count * 8;
    // CUB's item counts are int: graphs beyond INT_MAX vertices keep their numbering
    if (n > 0x7FFFFFFFu) return SSSP_OK;
    unsigned* indeg = nullptr;
    CK(cudaMalloc(&indeg, (size_t)n * 4), "relabel: in-degrees");
    unsigned mx = 0;
    {
        unsigned* d_mx = nullptr;
        void* tmp = nullptr;
        size_t tb = 0;
        cudaError_t e = cudaMemset(indeg, 0, (size_t)n * 4);
        if (e == cudaSuccess) {
            indegree_kernel<<<aux_grid, 256>>>(g->d_adj, m, indeg);
            e = cudaGetLastError();
        }
        if (e == cudaSuccess) e = cub::DeviceReduce::Max(tmp, tb, indeg, d_mx, (int)n);
        if (e == cudaSuccess) e = cudaMalloc(&d_mx, 4);
        if (e == cudaSuccess) e = cudaMalloc(&tmp, tb);
        if (e == cudaSuccess) e = cub::DeviceReduce::Max(tmp, tb, indeg, d_mx, (int)n);
        if (e == cudaSuccess) e = cudaMemcpy(&mx, d_mx, 4, cudaMemcpyDeviceToHost);
        cudaFree(tmp);
        cudaFree(d_mx);
        if (e != cudaSuccess) {
            cudaFree(indeg);
            return cuda_fail(e, "relabel: max in-degree");
        }
    }
    g->max_indeg = mx;
    bool on = (double)mx > 64.0 * (double)m / (double)n;
    if (o.flags & SSSP_FLAG_RELABEL) on = true;
    if (o.flags & SSSP_FLAG_NO_RELABEL) on = false;
    if (!on) {
        cudaFree(indeg);
        return SSSP_OK;
    }
    unsigned *key = nullptr, *key_out = nullptr, *iota = nullptr, *old_of_new = nullptr, *new_of_old = nullptr;
    unsigned long long *deg_new = nullptr, *off_new = nullptr;
    uint2* adj_new = nullptr;
    void* tmp = nullptr;
    size_t tb_sort = 0, tb_scan = 0;
    auto cleanup = [&]() {
        cudaFree(indeg); cudaFree(key); cudaFree(key_out); cudaFree(iota); cudaFree(old_of_new);
        cudaFree(deg_new); cudaFree(tmp);
    };
    cudaError_t e = cudaSuccess;
    if (e == cudaSuccess) e = cudaMalloc(&key, (size_t)n * 4);
    if (e == cudaSuccess) e = cudaMalloc(&key_out, (size_t)n * 4);
    if (e == cudaSuccess) e = cudaMalloc(&iota, (size_t)n * 4);
    if (e == cudaSuccess) e = cudaMalloc(&old_of_new, (size_t)n * 4);
    if (e == cudaSuccess) e = cudaMalloc(&new_of_old, (size_t)n * 4);
    if (e == cudaSuccess) e = cudaMalloc(&deg_new, (size_t)(n + 1) * 8);
    if (e == cudaSuccess) e = cudaMalloc(&off_new, (size_t)(n + 1) * 8);
    if (e == cudaSuccess) e = cudaMalloc(&adj_new, (size_t)m * sizeof(uint2));
    if (e == cudaSuccess) e = cub::DeviceRadixSort::SortPairs(nullptr, tb_sort, key, key_out, iota, old_of_new, (int)n);
    if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(nullptr, tb_scan, deg_new, off_new, (int)n + 1);
    if (e == cudaSuccess) e = cudaMalloc(&tmp, std::max(tb_sort, tb_scan));
    if (e == cudaSuccess) {
        relabel_keys_kernel<<<aux_grid, 256>>>(indeg, n, key, iota);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cub::DeviceRadixSort::SortPairs(tmp, tb_sort, key, key_out, iota, old_of_new, (int)n);
    if (e == cudaSuccess) e = cudaMemset(deg_new + n, 0, 8);
    if (e == cudaSuccess) {
        relabel_inverse_kernel<<<aux_grid, 256>>>(old_of_new, n, g->d_off, new_of_old, deg_new);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(tmp, tb_scan, deg_new, off_new, (int)n + 1);
    if (e == cudaSuccess) {
        relabel_arcs_kernel<<<aux_grid, 256>>>(old_of_new, new_of_old, n, g->d_off, off_new, g->d_adj, adj_new);
        e = cudaDeviceSynchronize();
    }
    if (e == cudaSuccess) {
        g->h_perm.resize(n);
        e = cudaMemcpy(g->h_perm.data(), new_of_old, (size_t)n * 4, cudaMemcpyDeviceToHost);
    }
    cleanup();
    if (e != cudaSuccess) {
        g->h_perm.clear();
        cudaFree(new_of_old); cudaFree(off_new); cudaFree(adj_new);
        return cuda_fail(e, "relabeling the graph");
    }
    cudaFree(g->d_off);
    cudaFree(g->d_adj);
    g->d_off = off_new;
    g->d_adj = adj_new;
    g->d_perm = new_of_old;
    return SSSP_OK;
}

sssp_status create_impl(uint32_t n, uint64_t m, const uint64_t* row_offsets, const uint32_t* col, const uint32_t* w,
                        bool f32, const sssp_options* opts, sssp_graph** out) {
    if (!out) return fail(SSSP_ERR_INVALID_ARGUMENT, "out is NULL");
    *out = nullptr;
    if (!row_offsets || (m && (!col || !w))) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL CSR array");
    if (n == 0 || n > 0xFFFFFFFEu) return fail(SSSP_ERR_INVALID_ARGUMENT, "n must be in [1, 2^32-2]");
    sssp_options o;
    if (opts) o = *opts;
    else sssp_options_default(&o);
    sssp_status st = check_options(o);
    if (st) return st;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return fail(SSSP_ERR_NO_DEVICE, "no CUDA device");
    }
    if (o.device < 0 || o.device >= ndev) return fail(SSSP_ERR_INVALID_ARGUMENT, "device ordinal out of range");
    cudaDeviceProp prop{};
    CK(cudaGetDeviceProperties(&prop, o.device), "device properties");
    if (prop.major != 10) return fail(SSSP_ERR_NO_DEVICE, std::string("built for sm_100a, device is ") + prop.name);
    DeviceGuard dg(o.device);

    sssp_graph* g = new sssp_graph();
    g->device = o.device;
    g->n = n;
    g->m = m;
    g->opts = o;
    g->sm_count = prop.multiProcessorCount;
    g->f32 = f32;
    g->persist_max = prop.persistingL2CacheMaxSize > 0 ? (size_t)prop.persistingL2CacheMaxSize : 0;
    auto bail = [&](sssp_status s2) {
        sssp_graph_destroy(g);
        return s2;
    };
#define CKG(call, what)                                      \
    do {                                                     \
        cudaError_t e_ = (call);                             \
        if (e_ != cudaSuccess) return bail(cuda_fail(e_, what)); \
    } while (0)

    CKG(cudaMalloc(&g->d_off, (size_t)(n + 1) * 8), "allocating row_offsets");
    CKG(cudaMemcpy(g->d_off, row_offsets, (size_t)(n + 1) * 8, cudaMemcpyDefault), "copying row_offsets");
    unsigned long long ends[2] = {0, 0};
    CKG(cudaMemcpy(&ends[0], g->d_off, 8, cudaMemcpyDeviceToHost), "reading row_offsets[0]");
    CKG(cudaMemcpy(&ends[1], g->d_off + n, 8, cudaMemcpyDeviceToHost), "reading row_offsets[n]");
    if (ends[0] != 0) return bail(fail(SSSP_ERR_INVALID_GRAPH, "row_offsets[0] != 0 (index 0)"));
    if (ends[1] != m) return bail(fail(SSSP_ERR_INVALID_GRAPH, "row_offsets[n] != m (index " + std::to_string(n) + ")"));

    CKG(cudaMalloc(&g->d_adj, std::max<size_t>(m, 1) * sizeof(uint2)), "allocating arcs");
    CKG(cudaMalloc(&g->scratch.p, 64), "scratch");
    unsigned long long* d_bad = (unsigned long long*)g->scratch.p;  // [0],[1] bad idx, [2] sum_w, [3] max_w
    unsigned long long init_scr[5] = {~0ull, ~0ull, 0, 0, ~0ull};  // [4] first bad float weight
    CKG(cudaMemcpy(d_bad, init_scr, sizeof(init_scr), cudaMemcpyHostToDevice), "scratch init");
    const unsigned aux_grid = (unsigned)g->sm_count * 8;
    if (m) {
        unsigned *d_col = nullptr, *d_w = nullptr;
        CKG(cudaMalloc(&d_col, m * 4), "allocating col staging");
        cudaError_t e = cudaMalloc(&d_w, m * 4);
        if (e != cudaSuccess) {
            cudaFree(d_col);
            return bail(cuda_fail(e, "allocating w staging"));
        }
        e = cudaMemcpy(d_col, col, m * 4, cudaMemcpyDefault);
        if (e == cudaSuccess) e = cudaMemcpy(d_w, w, m * 4, cudaMemcpyDefault);
        if (e == cudaSuccess) {
            validate_csr_kernel<<<aux_grid, 256>>>(g->d_off, d_col, n, m, d_bad);
            if (f32)
                interleave_f32_kernel<<<aux_grid, 256>>>(d_col, d_w, g->d_adj, m, d_bad + 4, (unsigned*)(d_bad + 3));
            else
                interleave_kernel<<<aux_grid, 256>>>(d_col, d_w, g->d_adj, m, d_bad + 2, (unsigned*)(d_bad + 3));
            e = cudaDeviceSynchronize();
        }
        cudaFree(d_col);
        cudaFree(d_w);
        if (e != cudaSuccess) return bail(cuda_fail(e, "validating / interleaving the CSR"));
    } else {
        validate_csr_kernel<<<aux_grid, 256>>>(g->d_off, nullptr, n, 0, d_bad);
        CKG(cudaDeviceSynchronize(), "validating the CSR");
    }
    unsigned long long scr[5];
    CKG(cudaMemcpy(scr, d_bad, sizeof(scr), cudaMemcpyDeviceToHost), "reading validation result");
    if (scr[0] != ~0ull)
        return bail(fail(SSSP_ERR_INVALID_GRAPH, "row_offsets decreasing at index " + std::to_string(scr[0])));
    if (scr[1] != ~0ull)
        return bail(fail(SSSP_ERR_INVALID_GRAPH, "col[" + std::to_string(scr[1]) + "] >= n"));
    if (scr[4] != ~0ull)
        return bail(fail(SSSP_ERR_INVALID_GRAPH, "w[" + std::to_string(scr[4]) + "] is negative or NaN"));
    g->sum_w = scr[2];
    g->max_w = (uint32_t)scr[3];
    if (m) {
        sssp_status rs = relabel_graph(g, o);
        if (rs) return bail(rs);
    }
    if (m < (1ull << 32) && n) {
        CKG(cudaMalloc(&g->d_rows, (size_t)n * sizeof(uint2)), "allocating row records");
        rows32_kernel<<<aux_grid, 256>>>(g->d_off, n, g->d_rows);
        CKG(cudaDeviceSynchronize(), "building row records");
    }
    // initial Delta (reading R3): max_w / D (Meyer-Sanders' Theta(1/d) rule for Delta-stepping [15]),
    // or the Near-Far rule C * W / D with W = average weight, D = average degree, C = 32
    if (m && g->sum_w && !f32) {
        const double W = (double)g->sum_w / (double)m, D = (double)m / (double)n;
        g->heur_k_nf = std::min(ilog2_round(32.0 * W / D), 63u);
        g->heur_k_md = std::min(ilog2_round((double)g->max_w / std::max(D, 1.0)), 63u);
    }
    g->heur_k_span = std::min(ilog2_round((double)g->max_w / (double)o.num_buckets), 63u);
    // 32-bit distances are provably safe when (n-1) * max_w < 2^32 - 1; otherwise
    // they are tried first and the overflow flag triggers a 64-bit re-run.
    g->cur_bits = 32;

    for (auto& e : g->bev) CKG(cudaEventCreate(&e), "creating events");
    sssp_status st2 = ensure_slots(g, 1);
    if (st2) return bail(st2);
#undef CKG
    *out = g;
    return SSSP_OK;
}
}  // namespace

extern "C" {

sssp_status sssp_graph_create(uint32_t n, uint64_t m, const uint64_t* row_offsets, const uint32_t* col,
                              const uint32_t* w, const sssp_options* opts, sssp_graph** out) {
    return create_impl(n, m, row_offsets, col, w, false, opts, out);
}

sssp_status sssp_graph_create_f32(uint32_t n, uint64_t m, const uint64_t* row_offsets, const uint32_t* col,
                                  const float* w, const sssp_options* opts, sssp_graph** out) {
    return create_impl(n, m, row_offsets, col, (const uint32_t*)w, true, opts, out);
}

sssp_status sssp_graph_destroy(sssp_graph* g) {
    if (!g) return SSSP_OK;
    DeviceGuard dg(g->device);
    cudaDeviceSynchronize();
    if (g->copy_stream) cudaStreamDestroy(g->copy_stream);
    if (g->d_off) cudaFree(g->d_off);
    if (g->d_adj) cudaFree(g->d_adj);
    if (g->d_rows) cudaFree(g->d_rows);
    if (g->d_perm) cudaFree(g->d_perm);
    for (Workspace* w : g->ws) {
        w->release();
        delete w;
    }
    g->ws.clear();
    g->scratch.release();
    g->hostout.release();
    g->cert.release();
    for (auto& e : g->bev)
        if (e) cudaEventDestroy(e);
    delete g;
    return SSSP_OK;
}

sssp_status sssp_set_options(sssp_graph* g, const sssp_options* opts) {
    if (!g || !opts) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL argument");
    if (g->busy || g->async_pending) return fail(SSSP_ERR_BUSY, "a run is in flight");
    sssp_status st = check_options(*opts);
    if (st) return st;
    if (opts->device != g->device) return fail(SSSP_ERR_INVALID_ARGUMENT, "the device of a graph cannot change");
    DeviceGuard dg(g->device);
    const bool ring_change = opts->num_buckets != g->opts.num_buckets || opts->ring_items != g->opts.ring_items ||
                             ((opts->flags ^ g->opts.flags) & SSSP_FLAG_CHUNKED_RING);
    g->opts = *opts;
    if (opts->dist_bits) g->cur_bits = (int)opts->dist_bits;
    else g->cur_bits = 32;
    if (ring_change) {
        for (Workspace* w : g->ws) {
            w->ring.release();
            w->cap = 0;
        }
    }
    return SSSP_OK;
}

sssp_status sssp_run(sssp_graph* g, uint32_t source, uint64_t* dist_out, sssp_stream_t stream) {
    return run_many(g, &source, 1, dist_out, false, stream);
}

sssp_status sssp_run_batch(sssp_graph* g, const uint32_t* sources, uint32_t k, uint64_t* dist_out,
                           sssp_stream_t stream) {
    return run_many(g, sources, k, dist_out, false, stream);
}

sssp_status sssp_run_f32(sssp_graph* g, uint32_t source, float* dist_out, sssp_stream_t stream) {
    return run_many(g, &source, 1, dist_out, true, stream);
}

sssp_status sssp_run_batch_f32(sssp_graph* g, const uint32_t* sources, uint32_t k, float* dist_out,
                               sssp_stream_t stream) {
    return run_many(g, sources, k, dist_out, true, stream);
}

sssp_status sssp_get_stats(sssp_graph* g, sssp_stats* out) {
    if (!g || !out) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL argument");
    if (g->async_pending) {
        DeviceGuard dg(g->device);
        g->async_pending = false;
        Workspace& w = *g->ws[0];
        cudaError_t e = cudaEventSynchronize(w.ev[3]);
        if (e != cudaSuccess) return cuda_fail(e, "async run");
        // the status copy was enqueued after ev[3] on the same stream
        e = cudaDeviceSynchronize();
        if (e != cudaSuccess) return cuda_fail(e, "async run");
        const unsigned status = w.h_ctl->status;
        restore_persist(g);
        if (status) {
            // same cleanup and retry decisions as the synchronous path (settle_attempt):
            // the next run starts from a clean ring / chunk queue, 64-bit after an overflow
            sssp_status cst = clear_after_abort(w, (cudaStream_t)0);
            if (cst) return cst;
            if ((status & kStDistOverflow) && !g->opts.dist_bits) g->cur_bits = 64;
            if ((status & kStRingOverflow) && !(status & (kStTimeout | kStBug))) {
                // grow like the synchronous retry would, so the caller's re-run fits
                sssp_status gst = ensure_tasks(g, w, w.tcap * 2);
                if (gst == SSSP_OK) {
                    const unsigned long long ncap = w.cap * 2;
                    const int ib = w.ring_item_bytes;
                    w.ring.release();
                    gst = ensure_ring(g, w, ib, ncap);
                }
                if (gst) return gst;
            }
            g->stats.status = (status & kStRingOverflow)   ? SSSP_ERR_WORKLIST_OVERFLOW
                              : (status & kStTimeout)      ? SSSP_ERR_TIMEOUT
                              : (status & kStDistOverflow) ? SSSP_ERR_INVALID_ARGUMENT
                                                           : SSSP_ERR_CUDA;
            *out = g->stats;
            return fail((sssp_status)g->stats.status, "async run failed (status bits " + std::to_string(status) + ")");
        }
        accumulate(g, w, *w.h_ctl, (int)g->stats.dist_bits);
        g->stats.status = SSSP_OK;
    }
    *out = g->stats;
    return SSSP_OK;
}

sssp_status sssp_get_trace(sssp_graph* g, sssp_trace_entry* out, uint32_t cap, uint32_t* count) {
    if (!g || !count || (cap && !out)) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL argument");
    *count = 0;
    Workspace& w = *g->ws[0];
    if (!w.trace.p) return SSSP_OK;
    const uint32_t nvalid = std::min<uint32_t>(g->stats.trace_entries, w.trace_alloc);
    const uint32_t c = std::min(cap, nvalid);
    if (c) {
        DeviceGuard dg(g->device);
        CK(cudaMemcpy(out, w.trace.p, (size_t)c * sizeof(sssp_trace_entry), cudaMemcpyDeviceToHost), "trace copy");
    }
    *count = c;
    return SSSP_OK;
}

sssp_status sssp_get_profile(sssp_graph* g, uint64_t* out, uint32_t cap, uint32_t* count) {
    if (!g || !count || (cap && !out)) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL argument");
    const uint32_t c = std::min<uint32_t>(cap, kProfCounters);
    const Ctl* hc = g->ws.empty() ? nullptr : g->ws[0]->h_ctl;
    for (uint32_t i = 0; i < c; ++i) out[i] = hc ? hc->prof[i] : 0;
    *count = c;
    return SSSP_OK;
}

sssp_status sssp_certify(sssp_graph* g, uint32_t source, const void* dist, sssp_certificate* out,
                         sssp_stream_t stream) {
    if (!g || !dist || !out) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL argument");
    if (source >= g->n) return fail(SSSP_ERR_INVALID_ARGUMENT, "source >= n");
    if (g->busy || g->async_pending) return fail(SSSP_ERR_BUSY, "a run is in flight on this handle");
    DeviceGuard dg(g->device);
    std::memset(out, 0, sizeof(*out));
    cudaStream_t s = (cudaStream_t)stream;
    const size_t esz = g->f32 ? 4 : 8;
    bool is_dev = false;
    sssp_status st = classify_out(g, dist, &is_dev);
    if (st) return st;
    if (!is_dev) {  // host vector: stage it on the device
        if (!g->hostout.p) {
            CK(cudaMalloc(&g->hostout.p, (size_t)g->n * 8), "allocating the staging buffer");
            g->hostout.bytes = (size_t)g->n * 8;
        }
        CK(cudaMemcpyAsync(g->hostout.p, dist, (size_t)g->n * esz, cudaMemcpyHostToDevice, s), "staging dist");
        dist = g->hostout.p;
    }
    if (!g->cert.p) {
        CK(cudaMalloc(&g->cert.p, sizeof(CertState)), "allocating the certificate state");
        g->cert.bytes = sizeof(CertState);
    }
    CertState h{};
    h.first_violated = h.first_unanchored = ~0ull;
    CK(cudaMemcpyAsync(g->cert.p, &h, sizeof(h), cudaMemcpyHostToDevice, s), "certificate state");
    Workspace& w = *g->ws[0];
    unsigned long long* dint = (unsigned long long*)w.dist.p;  // 8n bytes of scratch (no run in flight)
    unsigned* anchors = (unsigned*)w.expanded.p;              // n bits
    CertState* dst = (CertState*)g->cert.p;
    const unsigned src_int = g->h_perm.empty() ? source : g->h_perm[source];
    const unsigned grid = (unsigned)g->sm_count * 8;
    auto run_rounds = [&](auto kf) -> sssp_status {
        constexpr bool kF = decltype(kf)::value;
        certify_scatter_kernel<kF><<<grid, 256, 0, s>>>(dist, dint, g->d_perm, g->n, source, anchors, dst);
        certify_arcs_kernel<kF><<<grid, 256, 0, s>>>(dint, g->d_off, g->d_adj, g->n, src_int, anchors, dst);
        CK(cudaGetLastError(), "certificate kernels");
        CK(cudaMemcpyAsync(&h, dst, sizeof(h), cudaMemcpyDeviceToHost, s), "certificate state");
        CK(cudaStreamSynchronize(s), "certificate");
        // tight arcs between equal distances: anchor to a fixed point (at most n rounds)
        if (h.equal_tight) {
            for (uint32_t r = 0; r < g->n; ++r) {
                CK(cudaMemsetAsync(&dst->changed, 0, 8, s), "certificate flag");
                certify_equal_kernel<kF><<<grid, 256, 0, s>>>(dint, g->d_off, g->d_adj, g->n, anchors, dst);
                CK(cudaMemcpyAsync(&h, dst, sizeof(h), cudaMemcpyDeviceToHost, s), "certificate state");
                CK(cudaStreamSynchronize(s), "certificate");
                out->fixpoint_rounds = r + 1;
                if (!h.changed) break;
            }
        }
        certify_check_kernel<kF><<<grid, 256, 0, s>>>(dint, g->d_off, g->n, anchors, dst);
        CK(cudaGetLastError(), "certificate kernels");
        CK(cudaMemcpyAsync(&h, dst, sizeof(h), cudaMemcpyDeviceToHost, s), "certificate state");
        CK(cudaStreamSynchronize(s), "certificate");
        return SSSP_OK;
    };
    st = g->f32 ? run_rounds(std::true_type{}) : run_rounds(std::false_type{});
    if (st) return st;
    auto to_caller = [&](unsigned long long iv) -> uint64_t {
        if (iv == ~0ull || g->h_perm.empty()) return iv;
        for (uint32_t v = 0; v < g->n; ++v)
            if (g->h_perm[v] == iv) return v;
        return iv;
    };
    out->source_ok = h.source_bad == 0 ? 1u : 0u;
    out->violated_arcs = h.violated;
    out->first_violated_tail = to_caller(h.first_violated);
    out->unanchored = h.unanchored;
    out->first_unanchored = to_caller(h.first_unanchored);
    out->bad_markers = h.bad_inf;
    out->reachable = h.reach_v;
    out->reach_edges = h.reach_e;
    out->exact = (out->source_ok && !h.violated && !h.unanchored && !h.bad_inf) ? 1u : 0u;
    return SSSP_OK;
}

sssp_status sssp_graph_info(const sssp_graph* g, uint32_t* n, uint64_t* m, uint64_t* sum_w, uint32_t* max_w,
                            uint32_t* heuristic_delta_log2) {
    if (!g) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL graph");
    if (n) *n = g->n;
    if (m) *m = g->m;
    if (sum_w) *sum_w = g->sum_w;
    if (max_w) *max_w = g->max_w;
    if (heuristic_delta_log2) *heuristic_delta_log2 = heuristic_k(g);
    return SSSP_OK;
}

sssp_status sssp_graph_layout(const sssp_graph* g, uint32_t* relabeled, uint32_t* max_indeg) {
    if (!g) return fail(SSSP_ERR_INVALID_ARGUMENT, "NULL graph");
    if (relabeled) *relabeled = g->d_perm ? 1u : 0u;
    if (max_indeg) *max_indeg = g->max_indeg;
    return SSSP_OK;
}

uint32_t sssp_bucket_offset(uint64_t d, uint32_t delta_log2, uint64_t head, uint32_t num_buckets) {
    if (num_buckets < 1) return 0;
    return adds_bucket_offset(d, delta_log2, head, num_buckets);
}

const char* sssp_status_string(sssp_status st) {
    switch (st) {
        case SSSP_OK: return "SSSP_OK";
        case SSSP_ERR_INVALID_ARGUMENT: return "SSSP_ERR_INVALID_ARGUMENT";
        case SSSP_ERR_INVALID_GRAPH: return "SSSP_ERR_INVALID_GRAPH";
        case SSSP_ERR_OUT_OF_MEMORY: return "SSSP_ERR_OUT_OF_MEMORY";
        case SSSP_ERR_CUDA: return "SSSP_ERR_CUDA";
        case SSSP_ERR_WORKLIST_OVERFLOW: return "SSSP_ERR_WORKLIST_OVERFLOW";
        case SSSP_ERR_TIMEOUT: return "SSSP_ERR_TIMEOUT";
        case SSSP_ERR_DEVICE_MISMATCH: return "SSSP_ERR_DEVICE_MISMATCH";
        case SSSP_ERR_BUSY: return "SSSP_ERR_BUSY";
        case SSSP_ERR_NO_DEVICE: return "SSSP_ERR_NO_DEVICE";
    }
    return "SSSP_ERR_UNKNOWN";
}

const char* sssp_last_error(void) { return g_err.c_str(); }

#define SSSP_STR2(x) #x
#define SSSP_STR(x) SSSP_STR2(x)
const char* sssp_version(void) {
    return "adds-sssp 0.1 (sm_100a, CUDA " SSSP_STR(__CUDACC_VER_MAJOR__) "." SSSP_STR(__CUDACC_VER_MINOR__) ")";
}

}  // extern "C"

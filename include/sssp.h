/*
 * sssp.h -- C ABI of the B200-native ADDS single-source shortest-path library
 * (libsssp.so, built from paper_conf_ppopp_wangfl21_b200/csrc/).
 *
 * Reference: K. Wang, D. Fussell, C. Lin, "A Fast Work-Efficient SSSP Algorithm
 * for GPUs", PPoPP '21.  Citations "P:<line>" are lines of
 * /root/reference/PAPER.md; "§8(x)" are sections of SURVEY.md.
 *
 * The operation (§3 "Background"): for a directed graph with
 * non-negative edge weights and a source s, compute for every vertex v the
 * shortest distance from s:
 *     dist[v] = min over directed paths s ~> v of the sum of arc weights,
 *     dist[s] = 0,   dist[v] = UINT64_MAX  iff no path exists.
 * The method (§5) is ADDS -- asynchronous Delta-stepping with a
 * 32-bucket approximate priority queue and a run-time Delta controller.  The
 * schedule changes only the work performed, never the result, and all
 * arithmetic is integer, so results are bit-exact and deterministic.
 *
 * Conventions
 *  - Every entry point returns sssp_status; nothing throws across the ABI and
 *    nothing calls exit().  On error, sssp_last_error() returns a thread-local
 *    human-readable detail string (valid until the next call on that thread).
 *  - Graph: CSR with n vertices and m directed arcs.  row_offsets[n+1] (uint64,
 *    row_offsets[0]=0, non-decreasing, row_offsets[n]=m), col[m] (uint32,
 *    < n) and w[m] (uint32 weights, any value incl. 0).  Self-loops and
 *    parallel arcs are allowed.  n <= 2^32-2 (UINT32_MAX is a reserved id).
 *  - Pointers passed to sssp_graph_create may be host or device memory (detected
 *    with cudaPointerGetAttributes); the library COPIES them into its own
 *    device memory and the caller keeps ownership.
 *  - dist_out may be a device pointer on the graph's device (the fast path) or
 *    host memory (the library then copies the result back before returning).
 *  - Streams: work is enqueued on `stream` (NULL = legacy default stream).
 *    By default a run waits for its 64-byte status block so that device-side
 *    errors (worklist overflow, 32-bit distance overflow) can be handled
 *    (grow the ring / switch to 64-bit distances and re-run).  With
 *    SSSP_FLAG_ASYNC the call returns after enqueueing; the caller must
 *    synchronise the stream and then call sssp_get_stats() to learn the status.
 *  - Concurrency: at most one run in flight per handle (SSSP_ERR_BUSY).
 *    Distinct handles may run concurrently on distinct streams.
 */
#ifndef SSSP_H_
#define SSSP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Same underlying type as cudaStream_t (struct CUstream_st*). */
typedef struct CUstream_st *sssp_stream_t;

typedef enum sssp_status {
    SSSP_OK = 0,
    SSSP_ERR_INVALID_ARGUMENT = 1, /* NULL pointer, source >= n, k == 0, bad option */
    SSSP_ERR_INVALID_GRAPH = 2,    /* CSR validation failed; detail names the first bad index */
    SSSP_ERR_OUT_OF_MEMORY = 3,    /* device or pinned-host allocation failed */
    SSSP_ERR_CUDA = 4,             /* any other CUDA runtime error (detail has the CUDA string) */
    SSSP_ERR_WORKLIST_OVERFLOW = 5,/* bucket ring full and retries exhausted / NO_RETRY set */
    SSSP_ERR_TIMEOUT = 6,          /* device watchdog expired (options.timeout_ms) */
    SSSP_ERR_DEVICE_MISMATCH = 7,  /* dist_out lives on another device than the graph */
    SSSP_ERR_BUSY = 8,             /* a run is already in flight on this handle */
    SSSP_ERR_NO_DEVICE = 9         /* no CUDA device / not an sm_100 device */
} sssp_status;

/* Options.flags bits */
#define SSSP_FLAG_TRACE 0x1u     /* record Delta-controller samples into the trace ring (§5, Figs. 11-15 analog) */
#define SSSP_FLAG_ASYNC 0x2u     /* do not wait for the run's status block (see Streams above) */
#define SSSP_FLAG_NO_RETRY 0x4u  /* on worklist overflow return SSSP_ERR_WORKLIST_OVERFLOW instead of growing */
#define SSSP_FLAG_NO_LOCAL 0x8u  /* publish every child through the ring (ablation of CTA-local continuation) */
#define SSSP_FLAG_PROFILE 0x10u  /* accumulate per-phase SM-cycle counters (sssp_get_profile) */
#define SSSP_FLAG_NO_WARP_LOCAL 0x80u /* ablation: no warp-local continuation (a warp running its own
                                         head-bucket children hop after hop in the latency regime;
                                         default on when the average degree is <= 8) */
#define SSSP_FLAG_WARP_LOCAL 0x100u   /* force the warp-local continuation on whatever the degree */
#define SSSP_FLAG_FILTER16 0x200u     /* experiment (off by default, measured slower): filter relaxations
                                         with a 16-bit upper-bound array of dist (half its L2 footprint)
                                         instead of a load of dist itself; D11 */
#define SSSP_FLAG_RELABEL 0x400u      /* force the locality relabeling of the graph at create time (vertices
                                         renumbered by descending in-degree inside the library; inputs and
                                         outputs stay in the caller's numbering; D15) */
#define SSSP_FLAG_NO_RELABEL 0x800u   /* never relabel (default: relabel when max in-degree > 64 x average) */
#define SSSP_FLAG_ADAPT_ACTIVE 0x40u  /* (the default since round 2; kept for source compatibility) the
                                        controller varies the number of active buckets between
                                        the degree-based default A0 and 2*A0 from the CTAs holding work */
#define SSSP_FLAG_FIXED_ACTIVE 0x1000u /* ablation: keep the active-bucket count at its initial value */
#define SSSP_FLAG_CHUNKED_RING 0x2000u /* bucket storage as a shared pool of 4096-item chunks (the paper's
                                        block pool): memory bounded by the items alive at
                                        once (default pool 2n items, grown x2 on exhaustion) instead of
                                        one no-lap array of >= n items per bucket (32n items) */
#define SSSP_FLAG_WIDE_ROWS 0x4000u /* the throughput build reads the 64-bit row offsets instead of its
                                       32-bit row records {begin, degree} -- the path graphs with
                                       m >= 2^32 take (no records are built for them); for tests and
                                       ablations */
#define SSSP_FLAG_L2_PERSIST 0x20u /* reserve the L2 persisting set-aside for dist (raises the device-wide
                                     cudaLimitPersistingL2CacheSize to min(dist bytes, maximum)) and mark
                                     dist accesses evict_last.  Off by default: measured on B200
                                     (tools/l2_residency_bench.cu) it shrinks the normal L2 and LOWERS
                                     random-gather throughput (213 vs 263 G/s next to a 4 GB stream) */

/* Worker granularity (options.worker).  The warp-granular worker of round 1 was an
 * ablation measured slower on every config (D12) and has been removed;
 * the value 2 is rejected with SSSP_ERR_INVALID_ARGUMENT. */
#define SSSP_WORKER_AUTO 0u
#define SSSP_WORKER_CTA 1u

/* Algorithms (options.algorithm) */
#define SSSP_ALGO_ADDS 0u
#define SSSP_ALGO_NEAR_FAR 1u

/* Initial-Delta heuristics (options.delta_heuristic) */
#define SSSP_DELTA_H_RING_SPAN 0u
#define SSSP_DELTA_H_MAXW_OVER_D 2u
#define SSSP_DELTA_H_NEARFAR 1u

/* Delta modes */
#define SSSP_DELTA_DYNAMIC 0u    /* ADDS: run-time controller */
#define SSSP_DELTA_STATIC 1u     /* ablation "Static-Delta": keep delta_init for the whole run */

typedef struct sssp_options {
    uint32_t struct_size;      /* = sizeof(sssp_options); set by sssp_options_default */
    int32_t device;            /* CUDA device ordinal (default 0) */
    uint32_t num_buckets;      /* ring size B, power of two in [2, 32]; default 32 */
    uint32_t delta_mode;       /* SSSP_DELTA_DYNAMIC (default) or SSSP_DELTA_STATIC */
    uint64_t delta_init;       /* initial Delta; 0 = heuristic (see delta_heuristic) rounded to the
                                  nearest power of two; else rounded to a power of two */
    uint32_t clip_pct;         /* tail-bucket share that raises Delta and its floor; default 65 */
    uint32_t settle_head_switches; /* K controller steps (head switches or periodic steps) between Delta
                                      changes; default 8 */
    uint32_t util_lo_pct;      /* lower utilisation limit, % of resident threads; default 100 */
    uint32_t util_hi_pct;      /* upper utilisation limit, % of resident threads; default 400 */
    uint32_t waste_lo_permille;/* Delta may grow only while the recent re-expansion share is below this
                                  (default 500 = 50%) */
    uint32_t waste_hi_permille;/* Delta shrinks (not below its clip floor) while the share is above this
                                  (default 600 = 60%, i.e. ~2.5x Dijkstra's vertex work) */
    uint32_t period_us;        /* periodic controller step (default 20 us; head switches also step) */
    uint32_t delta_heuristic;  /* initial-Delta heuristic when delta_init == 0 ("a heuristic similar
                                  to the one described in Section 4.3"): SSSP_DELTA_H_RING_SPAN (default:
                                  max weight / num_buckets, so one maximum-weight hop from the head stays
                                  inside the ring -- the clipping argument of P:195), SSSP_DELTA_H_MAXW_OVER_D
                                  (max weight / average degree, Meyer-Sanders [15]) or SSSP_DELTA_H_NEARFAR
                                  (C * W / D with C = 32, the Near-Far rule of P:120) */
    uint32_t dist_bits;        /* 0 = auto (32-bit internal distances when provably or observably
                                  safe, else 64), 32 or 64 */
    uint64_t ring_items;       /* capacity of each bucket's circular array (items, rounded up to a
                                  power of two, >= 64); 0 = auto = max(2^16, next_pow2(n)).  With
                                  SSSP_FLAG_CHUNKED_RING: items of the shared chunk pool (>= 64
                                  chunks of 4096); 0 = auto = max(2^18, next_pow2(2n)) */
    uint32_t flags;            /* SSSP_FLAG_* */
    uint32_t block_threads;    /* worker CTA size: 0 = auto (512; 128 on road-like graphs), else 128/256/512/1024 */
    uint32_t grid_ctas;        /* 0 = every co-resident CTA; else at most this many CTAs */
    uint32_t batch_min;        /* minimum items a CTA claims when enough are available; 0 = auto
                                  (256 on the throughput build, 32 on road-like graphs) */
    uint32_t timeout_ms;       /* device watchdog (globaltimer); 0 = default 60000 */
    uint32_t trace_capacity;   /* trace ring entries when SSSP_FLAG_TRACE; 0 = 65536 */
    uint32_t active_init;      /* initial number of active (claimable) buckets; 0 = auto: 4 when
                                  the average degree is > 8 (CTAs take the next bucket's items instead
                                  of idling through the head bucket's tail), else 1 */
    uint32_t local_max;        /* head-bucket children a CTA keeps as its own next batch instead of
                                  publishing them, when its batch was at most half a CTA (latency regime);
                                  0 = auto = 128; see SSSP_FLAG_NO_LOCAL */
    uint32_t max_backoff_ns;   /* idle CTAs back off exponentially up to this (0 = auto = 2048; 512 on road-like graphs) */
    uint32_t startup_permille; /* the controller may not grow Delta before this share of the vertices
                                  has been expanded or 32 head switches have happened (start-up
                                  frontiers are always small); default 20 (2%) */
    uint32_t concurrent_sources; /* sssp_run_batch: sources in flight at once on this GPU (NEXT-1), each
                                  with its own workspace (dist, bucket ring, counters) and stream and
                                  1/c of the SMs; the CSR is shared.  0/1 = one at a time */
    uint32_t algorithm;        /* SSSP_ALGO_ADDS (default) or SSSP_ALGO_NEAR_FAR: the paper's comparison
                                  system as an ablation -- 2 buckets, static Delta (default the
                                  Near-Far rule C*W/D), bulk-synchronous double-buffered piles */
    uint32_t split_degree;     /* hub splitting (§8(a) A5 "CTA/edge-chunk bins"): an expanded vertex with
                                  more out-arcs than this is processed by its CTA for the first
                                  split_degree arcs while the rest is published as split_degree-arc
                                  chunks that idle CTAs claim before bucket items (charged to the
                                  vertex's bucket, so the head cannot pass it early); 0 = auto
                                  (8 x CTA size), UINT32_MAX = off */
    uint32_t worker;           /* unit of work of the ADDS persistent kernel: SSSP_WORKER_AUTO (0) =
                                  SSSP_WORKER_CTA (a CTA claims up to a CTA-sized batch, expands it
                                  cooperatively and keeps head-bucket children on chip) */
    uint32_t reserved2[1];
} sssp_options;

typedef struct sssp_stats {
    uint64_t vertices_processed; /* items expanded (not stale): the paper's work count */
    uint64_t edges_relaxed;      /* arcs scanned from expanded items */
    uint64_t pushes;             /* items pushed into the bucket ring (incl. the source) */
    uint64_t stale_skips;        /* popped items whose distance was already improved */
    uint64_t reachable;          /* vertices with finite distance  (= V_dij) */
    uint64_t reach_edges;        /* sum of out-degrees of reachable vertices (= E_dij, GTEPS numerator) */
    uint64_t max_dist;           /* largest finite distance (float32 graphs: its IEEE bit pattern) */
    uint32_t init_delta_log2;    /* log2 of the initial Delta */
    uint32_t final_delta_log2;   /* log2 of Delta when the run ended */
    uint32_t head_switches;      /* head-bucket advances */
    uint32_t delta_changes;      /* Delta adjustments by the controller */
    uint32_t retries;            /* re-runs after overflow (ring growth or 64-bit distances) */
    uint32_t dist_bits;          /* 32 or 64: internal distance width of the last attempt */
    uint32_t grid_ctas;          /* persistent-kernel CTAs launched */
    uint32_t block_threads;      /* threads per CTA */
    uint32_t runs;               /* sources covered by these stats (1 for sssp_run) */
    uint32_t trace_entries;      /* valid entries in the trace ring (capped at capacity) */
    float kernel_ms;             /* device time of the persistent kernel(s) (CUDA events) */
    float total_ms;              /* device time init + kernel + finalize (CUDA events) */
    uint32_t status;             /* sssp_status of the last run (for SSSP_FLAG_ASYNC) */
    float batch_ms;              /* device time of the whole call on the caller's stream (CUDA events) */
    uint32_t concurrency;        /* sources that were in flight at once */
    uint32_t worker;             /* SSSP_WORKER_CTA: the worker granularity that ran */
    uint64_t ring_bytes;         /* device bytes of one workspace's bucket storage (items + chunk
                                    tables); the run used max(1, concurrency) workspaces */
} sssp_stats;

/* One Delta-controller sample (written at each head-bucket switch and at each
 * periodic controller step). */
typedef struct sssp_trace_entry {
    uint64_t time_ns;        /* %globaltimer */
    uint64_t head;           /* absolute head bucket number */
    uint64_t pending_total;  /* items reserved but not completed, all buckets */
    uint64_t pending_window; /* same, active buckets only */
    uint64_t pending_tail;   /* same, tail (clip) bucket */
    uint32_t delta_log2;     /* Delta in force after the step */
    uint32_t active;         /* bits 0-7: active buckets after the step; bits 8-15: floor of log2 Delta
                                (the clip bound); bits 16-23: ceiling of log2 Delta (a value
                                measured wasteful, not grown into again; 255 = none) */
    uint32_t waste_permille; /* re-expansion share of recent expansions (work-waste signal) */
    uint32_t reason;         /* bits 0-7: 1 = head-bucket switch, 2 = periodic controller step;
                                bits 8-16: decision inputs (1 low util, 2 high util, 4 work beyond the
                                window, 8 wasteful, 16 frugal, 32 clipping, 64 waste known,
                                128 start-up over, 256 settled);
                                bits 20-29: share of recent pushes clipped into the tail (permille),
                                bit 30: that share is measured (>= 64K recent pushes) */
} sssp_trace_entry;

/* Opaque handle: owns the device CSR, the workspace (bucket ring, counters,
 * trace ring), a pinned status block and the timing events. */
typedef struct sssp_graph sssp_graph;

/* Fills *opts with the defaults documented above. NULL-safe. */
void sssp_options_default(sssp_options *opts);

/* Validates the CSR on the device (O(n+m)), copies it into library-owned
 * device memory (interleaved {col,w} arcs), computes the graph statistics
 * used for the initial Delta (sum of weights), and allocates the
 * run workspace on opts->device.  opts may be NULL (defaults).
 * Errors: INVALID_ARGUMENT (NULL out or arrays / n == 0 / n > 2^32-2),
 * INVALID_GRAPH (detail names the first offending index), OUT_OF_MEMORY,
 * NO_DEVICE, CUDA.  On error *out is set to NULL and nothing leaks. */
sssp_status sssp_graph_create(uint32_t n, uint64_t m, const uint64_t *row_offsets,
                              const uint32_t *col, const uint32_t *w,
                              const sssp_options *opts, sssp_graph **out);

/* Float32 weights (NEXT-3; the paper's float variant): w[m] are
 * non-negative IEEE binary32 values (-0.0 is folded into +0.0; a negative or NaN
 * weight is SSSP_ERR_INVALID_GRAPH with the first bad index; +inf arcs never
 * improve anything).  Distances are accumulated in binary32 with
 * round-to-nearest-even addition: dist[v] = min over paths of the left-to-right
 * float-rounded path sum (bit-exactly what a float Dijkstra computes).  Such a
 * handle is run with sssp_run_f32 / sssp_run_batch_f32 only. */
sssp_status sssp_graph_create_f32(uint32_t n, uint64_t m, const uint64_t *row_offsets,
                                  const uint32_t *col, const float *w,
                                  const sssp_options *opts, sssp_graph **out);

/* Releases everything the handle owns (synchronises its device first). NULL-safe. */
sssp_status sssp_graph_destroy(sssp_graph *g);

/* Replaces the run-time options of an existing handle (Delta mode/initial
 * Delta, controller constants, ring size, grid/block shape, flags).  The
 * device, and the CSR, cannot change.  Not allowed while a run is in flight. */
sssp_status sssp_set_options(sssp_graph *g, const sssp_options *opts);

/* Single-source run: dist_out[v] (uint64, n entries) = exact distance from
 * `source`, UINT64_MAX when unreachable.  Enqueued on `stream`; see
 * "Streams" for the synchronous default and SSSP_FLAG_ASYNC.
 * Errors: INVALID_ARGUMENT (source >= n, NULL dist_out), DEVICE_MISMATCH,
 * BUSY, WORKLIST_OVERFLOW (only with NO_RETRY or after 20 doublings), TIMEOUT,
 * CUDA. */
sssp_status sssp_run(sssp_graph *g, uint32_t source, uint64_t *dist_out, sssp_stream_t stream);

/* Multi-source batch: k sources (host array), results row-major
 * dist_out[i*n + v] for source i (k*n uint64 entries, device or host).
 * Equivalent to k calls of sssp_run (bit-identical); with
 * options.concurrent_sources = c > 1 up to c sources run concurrently (each
 * with its own workspace and stream, joined back to `stream` before return).
 * A host dist_out (pinned for full PCIe speed) is filled through two device
 * staging rows per slot (2*c*n*8 bytes, kept by the handle): each finished
 * row is copied on an internal copy stream while the next sources compute,
 * and every row is on the host when the call returns.
 * Stats cover the whole batch (batch_ms = device time of the call).  Errors as sssp_run plus
 * INVALID_ARGUMENT for k == 0 or any source >= n (checked before any work). */
sssp_status sssp_run_batch(sssp_graph *g, const uint32_t *sources, uint32_t k,
                           uint64_t *dist_out, sssp_stream_t stream);

/* Float32-weight runs: dist_out[v] (float, n entries; k*n for the batch), +inf
 * when unreachable.  Same stream / error semantics as sssp_run(_batch);
 * INVALID_ARGUMENT when the handle was created with integer weights. */
sssp_status sssp_run_f32(sssp_graph *g, uint32_t source, float *dist_out, sssp_stream_t stream);
sssp_status sssp_run_batch_f32(sssp_graph *g, const uint32_t *sources, uint32_t k,
                               float *dist_out, sssp_stream_t stream);

/* Statistics of the last run/batch (valid after the run's stream is
 * synchronised).  With SSSP_FLAG_ASYNC this also performs the deferred
 * status check and returns the run's status. */
sssp_status sssp_get_stats(sssp_graph *g, sssp_stats *out);

/* Copies up to `cap` trace entries of the last run (SSSP_FLAG_TRACE) into
 * host memory `out`; *count receives the number copied. */
sssp_status sssp_get_trace(sssp_graph *g, sssp_trace_entry *out, uint32_t cap, uint32_t *count);

/* Per-phase profile of the last run (SSSP_FLAG_PROFILE), summed over CTAs:
 * out[0..15] = cycles in claim (successful), idle (failed claim + advance +
 * backoff), pop, scan, rounds (expand/relax/stage), flush, complete, CTA
 * lifetime; then counts of ring batches, local batches, idle iterations,
 * flushes, rounds, CTAs; then cycles in arc-window setup (owner scan + async
 * arc prefetch) and the window count.  *count receives min(cap, 16). */
sssp_status sssp_get_profile(sssp_graph *g, uint64_t *out, uint32_t cap, uint32_t *count);

/* Certificate of a distance vector (SURVEY.md §8(c) "What pins each part"): the
 * O(n + m) checks that hold iff `dist` is the exact distance vector from `source`
 * -- (i) dist[source] = 0; (ii) no arc (u, v, w) with dist[u] finite has
 * dist[v] > dist[u] + w; (iii) every finite vertex is reachable from the source
 * through tight arcs (dist[u] + w == dist[v]); (iv) unreachable entries carry the
 * exact marker.  Float32-weight graphs use the IEEE round-to-nearest sum. */
typedef struct sssp_certificate {
    uint32_t exact;               /* 1 iff (i)-(iv) all hold */
    uint32_t source_ok;           /* (i) */
    uint64_t violated_arcs;       /* (ii): arcs whose head is above tail + weight */
    uint64_t first_violated_tail; /* caller id of the smallest violated arc tail (UINT64_MAX: none) */
    uint64_t unanchored;          /* (iii): finite vertices not reachable through tight arcs */
    uint64_t first_unanchored;    /* caller id of the smallest such vertex (UINT64_MAX: none) */
    uint64_t bad_markers;         /* (iv) float graphs: NaN / negative entries */
    uint64_t reachable;           /* finite entries (V_dij when exact) */
    uint64_t reach_edges;         /* sum of their out-degrees (E_dij when exact) */
    uint32_t fixpoint_rounds;     /* rounds spent on tight arcs between equal distances (0-weight arcs) */
    uint32_t reserved;
} sssp_certificate;

/* Checks `dist` (n entries in the caller's numbering: uint64 for integer graphs,
 * float for float32-weight graphs; device memory on the graph's device or host
 * memory) on the GPU with the certificate above: one pass over the arcs plus, only
 * when tight zero-weight arcs exist, a fixed point over them.  Synchronous on
 * `stream`; uses the handle's workspace as scratch, so not while a run is in flight
 * (BUSY).  The verdict is in *out (SSSP_OK means the check ran, not that it passed).
 * Errors: INVALID_ARGUMENT (NULL, source >= n), BUSY, DEVICE_MISMATCH, CUDA. */
sssp_status sssp_certify(sssp_graph *g, uint32_t source, const void *dist, sssp_certificate *out,
                         sssp_stream_t stream);

/* Graph facts: n, m, sum of weights, max weight, and the heuristic initial
 * Delta (log2) under options.delta_heuristic: round(log2(max_w / B)),
 * round(log2(max_w / D)) or round(log2(C * W / D)) with C = 32, W = sum_w/m,
 * D = m/n. */
sssp_status sssp_graph_info(const sssp_graph *g, uint32_t *n, uint64_t *m, uint64_t *sum_w,
                            uint32_t *max_w, uint32_t *heuristic_delta_log2);

/* Internal layout of the graph: *relabeled = 1 when the vertices were renumbered by
 * descending in-degree at create time (D15: locality of the gathered /
 * atomically updated distance array; sources and outputs always use the caller's
 * numbering), *max_indeg = the largest in-degree.  Either pointer may be NULL. */
sssp_status sssp_graph_layout(const sssp_graph *g, uint32_t *relabeled, uint32_t *max_indeg);

/* The bucket ring's priority mapping (§5.4-5.5), exposed for unit
 * tests: the ring offset (0 = head ... B-1 = tail) that an item of distance d
 * is pushed to when the head bucket is number `head` (absolute, in units of
 * Delta = 2^delta_log2) and the ring has B buckets: floor(d / Delta) - head,
 * clamped to [0, B-1] (items beyond the ring are clipped into the tail,
 * P:195).  Pure function, no device needed. */
uint32_t sssp_bucket_offset(uint64_t d, uint32_t delta_log2, uint64_t head, uint32_t num_buckets);

/* Static description strings. */
const char *sssp_status_string(sssp_status st);
const char *sssp_last_error(void);
/* Library build string (arch, version). */
const char *sssp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SSSP_H_ */

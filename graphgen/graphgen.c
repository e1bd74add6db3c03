/*
 * graphgen.c -- seeded synthetic CSR generators for the SSSP workloads.
 *
 * This module holds NO arithmetic of the SSSP method: it only builds input
 * graphs.  It is the one module shared by the oracle (oracle/) and the CUDA
 * path (paper_conf_ppopp_wangfl21_b200/); neither of those imports the other.
 *
 * Workload recipes:
 *   grid   : W x H 4-neighbour lattice, row-major ids, every directed arc has an
 *            independent weight U[lo,hi]   (configs 1 and 2; A19, A20)
 *   rmat   : Graph500 Kronecker, (a,b,c,d) = (0.57,0.19,0.19,0.05), 2^scale
 *            vertices, edge_factor * 2^scale directed arcs, duplicates and
 *            self-loops kept, ids relabelled by a seeded permutation (A18)
 *   er     : directed G(n, m) with iid uniform endpoints, duplicates and
 *            self-loops kept (A21)
 * Weights: w = lo + ((h >> 32) * (hi - lo + 1) >> 32) with h a counter-based
 * splitmix64 draw (A22), so the output does not depend on the thread count.
 *
 * CSR layout produced: row_offsets uint64[n+1], col uint32[m], w uint32[m];
 * each row sorted by (col, w) so parallel construction is deterministic.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---- counter-based RNG (splitmix64 finaliser over a keyed counter) ---- */
static inline uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
static inline uint64_t gg_key(uint64_t seed, uint64_t stream) {
    return mix64(seed * 0x9E3779B97F4A7C15ULL + 0x5851F42D4C957F2DULL + (stream << 40));
}
static inline uint64_t gg_draw(uint64_t key, uint64_t i) {
    return mix64(key + (i + 1) * 0x9E3779B97F4A7C15ULL);
}
/* uniform integer in [lo, hi] (inclusive), A22 */
static inline uint32_t gg_uniform(uint64_t h, uint32_t lo, uint32_t hi) {
    uint64_t span = (uint64_t)hi - lo + 1; /* <= 2^32 */
    return lo + (uint32_t)(((h >> 32) * span) >> 32);
}

uint64_t gg_hash(uint64_t seed, uint64_t stream, uint64_t i) {
    return gg_draw(gg_key(seed, stream), i);
}

enum { ST_GRID_W = 1, ST_RMAT_LVL = 2, ST_RMAT_PERM = 3, ST_RMAT_W = 4,
       ST_ER_EP = 5, ST_ER_W = 6, ST_SRC = 7, ST_FLOAT_W = 8 };

/* ------------------------------------------------------------------ grid */
/* number of arcs of a W x H 4-neighbour lattice */
uint64_t gg_grid_arcs(uint32_t W, uint32_t H) {
    return 2ULL * (uint64_t)H * (W - 1) + 2ULL * (uint64_t)W * (H - 1);
}

static inline uint32_t grid_deg(uint32_t r, uint32_t c, uint32_t W, uint32_t H) {
    return (r > 0) + (c > 0) + (c + 1 < W) + (r + 1 < H);
}

/* Fills off[n+1], col[m], w[m]; m must equal gg_grid_arcs(W,H). Returns 0. */
int gg_grid(uint32_t W, uint32_t H, uint32_t lo, uint32_t hi, uint64_t seed,
            uint64_t *off, uint32_t *col, uint32_t *w) {
    uint64_t n = (uint64_t)W * H;
    /* offsets: closed form per row of the lattice */
    off[0] = 0;
    for (uint64_t v = 0; v < n; ++v) {
        uint32_t r = (uint32_t)(v / W), c = (uint32_t)(v % W);
        off[v + 1] = off[v] + grid_deg(r, c, W, H);
    }
    uint64_t key = gg_key(seed, ST_GRID_W);
#pragma omp parallel for schedule(static)
    for (int64_t vv = 0; vv < (int64_t)n; ++vv) {
        uint64_t v = (uint64_t)vv;
        uint32_t r = (uint32_t)(v / W), c = (uint32_t)(v % W);
        uint64_t e = off[v];
        /* ascending column order: up, left, right, down */
        if (r > 0)     { col[e] = (uint32_t)(v - W); ++e; }
        if (c > 0)     { col[e] = (uint32_t)(v - 1); ++e; }
        if (c + 1 < W) { col[e] = (uint32_t)(v + 1); ++e; }
        if (r + 1 < H) { col[e] = (uint32_t)(v + W); ++e; }
        for (uint64_t k = off[v]; k < e; ++k) w[k] = gg_uniform(gg_draw(key, k), lo, hi);
    }
    return 0;
}

/* ------------------------------------------------- edge-list -> sorted CSR */
static int cmp_u64(const void *a, const void *b) {
    uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
    return (x > y) - (x < y);
}
static void sort_row(uint64_t *k, uint64_t len) {
    if (len < 32) { /* insertion sort */
        for (uint64_t i = 1; i < len; ++i) {
            uint64_t x = k[i]; uint64_t j = i;
            while (j > 0 && k[j - 1] > x) { k[j] = k[j - 1]; --j; }
            k[j] = x;
        }
    } else {
        qsort(k, len, sizeof(uint64_t), cmp_u64);
    }
}

typedef void (*arc_fn)(const void *ctx, uint64_t i, uint32_t *src, uint32_t *dst, uint32_t *wt);

/* Two-pass CSR build: count, prefix, scatter packed (dst<<32|w), sort rows. */
static int build_csr(uint64_t n, uint64_t m, arc_fn gen, const void *ctx,
                     uint64_t *off, uint32_t *col, uint32_t *w) {
    uint64_t *cnt = (uint64_t *)calloc(n + 1, sizeof(uint64_t));
    uint64_t *keys = (uint64_t *)malloc((m ? m : 1) * sizeof(uint64_t));
    if (!cnt || !keys) { free(cnt); free(keys); return -1; }
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)m; ++i) {
        uint32_t s, d, wt; gen(ctx, (uint64_t)i, &s, &d, &wt);
#pragma omp atomic
        cnt[s] += 1;
    }
    off[0] = 0;
    for (uint64_t v = 0; v < n; ++v) off[v + 1] = off[v] + cnt[v];
    memcpy(cnt, off, n * sizeof(uint64_t)); /* cursors */
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)m; ++i) {
        uint32_t s, d, wt; gen(ctx, (uint64_t)i, &s, &d, &wt);
        uint64_t pos;
#pragma omp atomic capture
        pos = cnt[s]++;
        keys[pos] = ((uint64_t)d << 32) | wt;
    }
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < (int64_t)n; ++v) {
        uint64_t b = off[v], e = off[v + 1];
        sort_row(keys + b, e - b);
        for (uint64_t k = b; k < e; ++k) { col[k] = (uint32_t)(keys[k] >> 32); w[k] = (uint32_t)keys[k]; }
    }
    free(cnt); free(keys);
    return 0;
}

/* ------------------------------------------------------------------ RMAT */
typedef struct { uint32_t scale; uint64_t klvl, kw; uint32_t lo, hi;
                 uint32_t ta, tab, tabc; const uint32_t *perm; } rmat_ctx;

static void rmat_arc(const void *vc, uint64_t i, uint32_t *src, uint32_t *dst, uint32_t *wt) {
    const rmat_ctx *c = (const rmat_ctx *)vc;
    uint32_t s = 0, d = 0;
    uint64_t h = 0;
    uint32_t per = (c->scale + 3) / 4; /* 16-bit draws, four per 64-bit hash */
    for (uint32_t l = 0; l < c->scale; ++l) {
        if ((l & 3) == 0) h = gg_draw(c->klvl, i * per + l / 4);
        uint32_t u = (uint32_t)(h & 0xFFFF); h >>= 16;
        uint32_t sb, db;
        if (u < c->ta) { sb = 0; db = 0; }
        else if (u < c->tab) { sb = 0; db = 1; }
        else if (u < c->tabc) { sb = 1; db = 0; }
        else { sb = 1; db = 1; }
        s = (s << 1) | sb; d = (d << 1) | db;
    }
    *src = c->perm[s]; *dst = c->perm[d];
    *wt = gg_uniform(gg_draw(c->kw, i), c->lo, c->hi);
}

/* Fisher-Yates permutation of [0,n) driven by the counter RNG (serial). */
static void seeded_perm(uint32_t *p, uint64_t n, uint64_t key) {
    for (uint64_t i = 0; i < n; ++i) p[i] = (uint32_t)i;
    for (uint64_t i = n; i > 1; --i) {
        uint64_t j = ((gg_draw(key, n - i) >> 32) * i) >> 32; /* uniform in [0, i) */
        uint32_t t = p[i - 1]; p[i - 1] = p[j]; p[j] = t;
    }
}

/* probabilities in 1/65536 units; graphgen.RMAT_ABC (37356,12452,12452; d=3276) ~ Graph500 */
int gg_rmat(uint32_t scale, uint32_t edge_factor, uint32_t pa, uint32_t pb, uint32_t pc,
            uint32_t lo, uint32_t hi, uint64_t seed, int permute,
            uint64_t *off, uint32_t *col, uint32_t *w) {
    uint64_t n = 1ULL << scale, m = (uint64_t)edge_factor << scale;
    uint32_t *perm = (uint32_t *)malloc(n * sizeof(uint32_t));
    if (!perm) return -1;
    if (permute) seeded_perm(perm, n, gg_key(seed, ST_RMAT_PERM));
    else for (uint64_t i = 0; i < n; ++i) perm[i] = (uint32_t)i;
    rmat_ctx c = { scale, gg_key(seed, ST_RMAT_LVL), gg_key(seed, ST_RMAT_W), lo, hi,
                   pa, pa + pb, pa + pb + pc, perm };
    int rc = build_csr(n, m, rmat_arc, &c, off, col, w);
    free(perm);
    return rc;
}

/* -------------------------------------------------------------------- ER */
typedef struct { uint64_t n; uint64_t kep, kw; uint32_t lo, hi; } er_ctx;
static void er_arc(const void *vc, uint64_t i, uint32_t *src, uint32_t *dst, uint32_t *wt) {
    const er_ctx *c = (const er_ctx *)vc;
    *src = (uint32_t)(((gg_draw(c->kep, 2 * i) >> 32) * c->n) >> 32);
    *dst = (uint32_t)(((gg_draw(c->kep, 2 * i + 1) >> 32) * c->n) >> 32);
    *wt = gg_uniform(gg_draw(c->kw, i), c->lo, c->hi);
}

int gg_er(uint64_t n, uint64_t m, uint32_t lo, uint32_t hi, uint64_t seed,
          uint64_t *off, uint32_t *col, uint32_t *w) {
    er_ctx c = { n, gg_key(seed, ST_ER_EP), gg_key(seed, ST_ER_W), lo, hi };
    return build_csr(n, m, er_arc, &c, off, col, w);
}

/* ------------------------------------------------------------- sources */
/* First k distinct seeded draws among vertices with out-degree >= 1 (A17).
 * Returns the number found (< k only if the graph has too few such vertices
 * or max_draws is exhausted). */
uint32_t gg_sources(uint64_t n, const uint64_t *off, uint64_t seed, uint32_t k,
                    uint32_t *out, uint64_t max_draws) {
    uint64_t key = gg_key(seed, ST_SRC);
    uint32_t got = 0;
    for (uint64_t j = 0; j < max_draws && got < k; ++j) {
        uint32_t v = (uint32_t)(((gg_draw(key, j) >> 32) * n) >> 32);
        if (off[v + 1] == off[v]) continue;
        int dup = 0;
        for (uint32_t t = 0; t < got; ++t) if (out[t] == v) { dup = 1; break; }
        if (!dup) out[got++] = v;
    }
    return got;
}

/* 64-bit fingerprint of a CSR (order-sensitive), for determinism checks */
uint64_t gg_fingerprint(uint64_t n, uint64_t m, const uint64_t *off, const uint32_t *col,
                        const uint32_t *w) {
    uint64_t h = mix64(n * 31 + m);
    /* chunked so it can run in parallel yet stay order sensitive */
    const uint64_t CH = 1 << 20;
    uint64_t nch = (m + CH - 1) / CH;
    uint64_t acc = 0;
#pragma omp parallel for reduction(^ : acc) schedule(static)
    for (int64_t c = 0; c < (int64_t)nch; ++c) {
        uint64_t b = (uint64_t)c * CH, e = b + CH < m ? b + CH : m, x = mix64((uint64_t)c + 1);
        for (uint64_t i = b; i < e; ++i) x = mix64(x ^ (((uint64_t)col[i] << 32) | w[i]));
        acc ^= mix64(x + (uint64_t)c);
    }
    uint64_t y = 0;
    for (uint64_t v = 0; v <= n; v += 1) y = mix64(y ^ off[v]) ;
    return mix64(h ^ acc ^ y);
}

int gg_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* float32 weights for an existing CSR (NEXT-3): w = lo + u * (hi - lo) with u a
 * 24-bit uniform in [0, 1) from the counter RNG (exactly representable), rounded
 * to binary32; independent of the integer weights. */
void gg_float_weights(uint64_t m, float lo, float hi, uint64_t seed, float *w) {
    uint64_t key = gg_key(seed, ST_FLOAT_W);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < (int64_t)m; ++e) {
        float u = (float)(gg_draw(key, (uint64_t)e) >> 40) * (1.0f / 16777216.0f);
        w[e] = lo + u * (hi - lo);
    }
}

/*
 * oracle.c -- CPU oracle for the SSSP hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (paper_conf_ppopp_wangfl21_b200/) never links, imports or calls it, and it
 * shares no code, header or helper with the CUDA path.
 *
 * What the method computes (§3 "Background"):
 *   "SSSP algorithms compute the shortest distance from a source vertex to
 *    every other vertex in a directed graph with non-negative edge weights ...
 *    initially set to infinity, this current shortest distance is refined
 *    until the shortest distance is found."
 * ADDS (§5) is a label-correcting Delta-stepping variant; buckets,
 * Delta, clipping, asynchrony and the controller change only the amount of
 * work, never the result.  So the oracle is the plain
 * definition
 *      dist[v] = min over directed paths s~>v of sum w(e)   (exact, uint64)
 *      dist[s] = 0,   dist[v] = UINT64_MAX iff v is unreachable,
 * computed by the paper's own serial baseline, binary-heap Dijkstra
 * (§6.1.2 "a highly tuned serial implementation of Dijkstra's algorithm
 * ... which implements the priority queue using a binary heap"), with lazy
 * deletion.  Its work counters follow the paper's work-efficiency definition
 * (§3.1: "the inverse of the total number of vertices processed"):
 *      V_dij = vertices processed (popped with a current distance),
 *      E_dij = arcs scanned from those vertices.
 *
 * oracle_certify() is the O(n+m) certificate of SURVEY.md §8(c) (complete for
 * w >= 0): (i) dist[s]=0; (ii) dist[v] <= dist[u]+w for every arc with finite
 * dist[u]; (iii) every finite v is reached from s through tight arcs
 * (dist[u]+w == dist[v]); (iv) non-finite values are exactly UINT64_MAX.
 *
 * Pins (tests/test_oracle.py, -m "not gpu"): hand-worked graphs
 * (tests/golden/), brute-force Bellman-Ford / Floyd-Warshall on tiny graphs,
 * closed forms (BFS hops, Manhattan distance, prefix sums, complete DAG),
 * scipy.sparse.csgraph.dijkstra, and the certificate's accept/reject
 * behaviour.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define INF UINT64_MAX

/* ------------------------------------------------ binary min-heap of (d, v) */
typedef struct { uint64_t d; uint32_t v; } item_t;
typedef struct { item_t *a; uint64_t size, cap; } heap_t;

static int heap_push(heap_t *h, uint64_t d, uint32_t v) {
    if (h->size == h->cap) {
        uint64_t nc = h->cap ? 2 * h->cap : 1024;
        item_t *na = (item_t *)realloc(h->a, nc * sizeof(item_t));
        if (!na) return -1;
        h->a = na; h->cap = nc;
    }
    uint64_t i = h->size++;
    while (i > 0) { /* sift up */
        uint64_t p = (i - 1) / 2;
        if (h->a[p].d <= d) break;
        h->a[i] = h->a[p]; i = p;
    }
    h->a[i].d = d; h->a[i].v = v;
    return 0;
}

static item_t heap_pop(heap_t *h) {
    item_t top = h->a[0];
    item_t last = h->a[--h->size];
    uint64_t i = 0, n = h->size;
    for (;;) { /* sift down */
        uint64_t l = 2 * i + 1, r = l + 1, c = l;
        if (l >= n) break;
        if (r < n && h->a[r].d < h->a[l].d) c = r;
        if (h->a[c].d >= last.d) break;
        h->a[i] = h->a[c]; i = c;
    }
    if (n) h->a[i] = last;
    return top;
}

/* Binary-heap Dijkstra (lazy deletion).  dist_out: uint64[n].
 * Returns 0, or -1 on bad arguments / out of memory. */
int oracle_dijkstra(uint64_t n, uint64_t m, const uint64_t *off, const uint32_t *col,
                    const uint32_t *w, uint32_t s, uint64_t *dist_out,
                    uint64_t *V_out, uint64_t *E_out) {
    (void)m;
    if (s >= n) return -1;
    for (uint64_t v = 0; v < n; ++v) dist_out[v] = INF;
    heap_t h = { 0, 0, 0 };
    uint64_t V = 0, E = 0;
    dist_out[s] = 0;
    if (heap_push(&h, 0, s)) return -1;
    while (h.size) {
        item_t it = heap_pop(&h);
        uint32_t u = it.v;
        if (it.d > dist_out[u]) continue; /* stale entry */
        V += 1;
        E += off[u + 1] - off[u];
        for (uint64_t e = off[u]; e < off[u + 1]; ++e) {
            uint32_t v = col[e];
            uint64_t nd = it.d + (uint64_t)w[e];
            if (nd < dist_out[v]) {
                dist_out[v] = nd;
                if (heap_push(&h, nd, v)) { free(h.a); return -1; }
            }
        }
    }
    free(h.a);
    if (V_out) *V_out = V;
    if (E_out) *E_out = E;
    return 0;
}

/* Certificate (see header).  Returns 0 if dist is the exact SSSP distance
 * vector, otherwise a positive code naming the first violated clause:
 *   1 dist[s] != 0;  2 an arc u->v with dist[v] > dist[u]+w (or overflow);
 *   3 a finite vertex not reachable through tight arcs.
 * *bad_out receives the offending vertex (or arc index for code 2). */
int oracle_certify(uint64_t n, uint64_t m, const uint64_t *off, const uint32_t *col,
                   const uint32_t *w, uint32_t s, const uint64_t *dist, uint64_t *bad_out) {
    (void)m;
    if (s >= n || dist[s] != 0) { if (bad_out) *bad_out = s; return 1; }
    for (uint64_t u = 0; u < n; ++u) {
        if (dist[u] == INF) continue;
        for (uint64_t e = off[u]; e < off[u + 1]; ++e) {
            uint64_t nd = dist[u] + (uint64_t)w[e];
            if (nd < dist[u] /* wrapped */ || dist[col[e]] > nd) { if (bad_out) *bad_out = e; return 2; }
        }
    }
    /* BFS from s over tight arcs; every finite vertex must be visited */
    uint8_t *seen = (uint8_t *)calloc(n, 1);
    uint32_t *q = (uint32_t *)malloc(n * sizeof(uint32_t));
    if (!seen || !q) { free(seen); free(q); return -1; }
    uint64_t qh = 0, qt = 0;
    seen[s] = 1; q[qt++] = s;
    while (qh < qt) {
        uint32_t u = q[qh++];
        for (uint64_t e = off[u]; e < off[u + 1]; ++e) {
            uint32_t v = col[e];
            if (!seen[v] && dist[u] + (uint64_t)w[e] == dist[v]) { seen[v] = 1; q[qt++] = v; }
        }
    }
    int rc = 0;
    for (uint64_t v = 0; v < n; ++v)
        if (dist[v] != INF && !seen[v]) { if (bad_out) *bad_out = v; rc = 3; break; }
    free(seen); free(q);
    return rc;
}

/* Reached-set work counts recomputed from a final distance vector:
 * V = #finite, E = sum of out-degrees of finite vertices. */
void oracle_reach_counts(uint64_t n, const uint64_t *off, const uint64_t *dist,
                         uint64_t *V_out, uint64_t *E_out) {
    uint64_t V = 0, E = 0;
    for (uint64_t v = 0; v < n; ++v)
        if (dist[v] != INF) { V += 1; E += off[v + 1] - off[v]; }
    *V_out = V; *E_out = E;
}

/* ---------------------------------------------------------------- float32 weights (NEXT-3)
 * The paper's float variant: non-negative float weights, distances
 * accumulated in float.  What is computed (reading R16 in DESIGN.md): the same
 * refinement dist[v] = min(dist[v], fl(dist[u] + w)) with fl = IEEE binary32
 * round-to-nearest-even addition, from dist[s] = 0, all others +infinity.
 * Since fl(x + w) >= x for w >= 0 and fl is monotone, Dijkstra's order is still
 * valid and the result is the minimum over paths of the left-to-right
 * float-rounded path sum.  Unreachable (or overflowing to +inf) = +inf. */
typedef struct { float d; uint32_t v; } fitem_t;
typedef struct { fitem_t *a; uint64_t size, cap; } fheap_t;

static int fheap_push(fheap_t *h, float d, uint32_t v) {
    if (h->size == h->cap) {
        uint64_t nc = h->cap ? 2 * h->cap : 1024;
        fitem_t *na = (fitem_t *)realloc(h->a, nc * sizeof(fitem_t));
        if (!na) return -1;
        h->a = na; h->cap = nc;
    }
    uint64_t i = h->size++;
    while (i > 0) {
        uint64_t p = (i - 1) / 2;
        if (h->a[p].d <= d) break;
        h->a[i] = h->a[p]; i = p;
    }
    h->a[i].d = d; h->a[i].v = v;
    return 0;
}

static fitem_t fheap_pop(fheap_t *h) {
    fitem_t top = h->a[0];
    fitem_t last = h->a[--h->size];
    uint64_t i = 0, n = h->size;
    for (;;) {
        uint64_t l = 2 * i + 1, r = l + 1, c = l;
        if (l >= n) break;
        if (r < n && h->a[r].d < h->a[l].d) c = r;
        if (h->a[c].d >= last.d) break;
        h->a[i] = h->a[c]; i = c;
    }
    if (n) h->a[i] = last;
    return top;
}

int oracle_dijkstra_f32(uint64_t n, uint64_t m, const uint64_t *off, const uint32_t *col,
                        const float *w, uint32_t s, float *dist_out, uint64_t *V_out, uint64_t *E_out) {
    (void)m;
    if (s >= n) return -1;
    const float inf = __builtin_inff();
    for (uint64_t v = 0; v < n; ++v) dist_out[v] = inf;
    fheap_t h = { 0, 0, 0 };
    uint64_t V = 0, E = 0;
    dist_out[s] = 0.0f;
    if (fheap_push(&h, 0.0f, s)) return -1;
    while (h.size) {
        fitem_t it = fheap_pop(&h);
        uint32_t u = it.v;
        if (it.d > dist_out[u]) continue;
        V += 1;
        E += off[u + 1] - off[u];
        for (uint64_t e = off[u]; e < off[u + 1]; ++e) {
            volatile float nd = it.d + w[e];  /* binary32 RN addition (SSE, no excess precision) */
            if (nd < dist_out[col[e]]) {
                dist_out[col[e]] = nd;
                if (fheap_push(&h, nd, col[e])) { free(h.a); return -1; }
            }
        }
    }
    free(h.a);
    if (V_out) *V_out = V;
    if (E_out) *E_out = E;
    return 0;
}

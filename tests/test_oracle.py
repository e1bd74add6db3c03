"""Pins for the CPU oracle (oracle/) -- nothing here needs a GPU.

The oracle is checked against things other than itself (SURVEY.md §8(c) "What
pins each part"): hand-worked fixtures (tests/golden/), brute force
(Floyd-Warshall, Bellman-Ford) on tiny graphs, closed forms (BFS hop count,
Manhattan distance, prefix sums, complete DAG), a library routine
(scipy.sparse.csgraph.dijkstra, exact in float64 below 2^53) and the
certificate's accept/reject behaviour.  Each is chosen so a plausible mistake
(dropped term, wrong sign/index, transposed operand, 32-bit truncation,
duplicate handling) fails at least one of them.
"""
import collections
import random

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import graphgen as gg
import oracle
from conftest import golden_names, load_golden

INF = (1 << 64) - 1


# ------------------------------------------------------------ brute force
def floyd_warshall(n, arcs):
    """Textbook all-pairs Floyd-Warshall over Python ints (exact)."""
    D = [[INF] * n for _ in range(n)]
    for i in range(n):
        D[i][i] = 0
    for u, v, w in arcs:
        if w < D[u][v]:
            D[u][v] = w
    for k in range(n):
        Dk = D[k]
        for i in range(n):
            dik = D[i][k]
            if dik == INF:
                continue
            Di = D[i]
            for j in range(n):
                if Dk[j] != INF and dik + Dk[j] < Di[j]:
                    Di[j] = dik + Dk[j]
    return D


def bellman_ford(n, arcs, s):
    """Textbook Bellman-Ford: n-1 rounds over every arc."""
    d = [INF] * n
    d[s] = 0
    for _ in range(max(n - 1, 1)):
        changed = False
        for u, v, w in arcs:
            if d[u] != INF and d[u] + w < d[v]:
                d[v] = d[u] + w
                changed = True
        if not changed:
            break
    return d


def bfs_hops(g, s):
    hops = [INF] * g.n
    hops[s] = 0
    q = collections.deque([s])
    off, col = g.row_offsets, g.col
    while q:
        u = q.popleft()
        for e in range(int(off[u]), int(off[u + 1])):
            v = int(col[e])
            if hops[v] == INF:
                hops[v] = hops[u] + 1
                q.append(v)
    return hops


arc_lists = st.integers(1, 20).flatmap(
    lambda n: st.tuples(
        st.just(n),
        st.lists(
            st.tuples(st.integers(0, n - 1), st.integers(0, n - 1),
                      st.one_of(st.integers(0, 9), st.integers(0, 1000), st.just(0xFFFFFFFF))),
            max_size=4 * n),
        st.integers(0, n - 1)))


# ------------------------------------------------------------ golden fixtures
@pytest.mark.parametrize("name", golden_names())
def test_golden_fixture(name):
    fx = load_golden(name)
    g = gg.from_arcs(fx["n"], fx["arcs"])
    dist, V, E = oracle.dijkstra(g, fx["source"])
    assert [int(x) for x in dist] == fx["dist"]
    assert V == fx["V"] and E == fx["E"]
    assert oracle.certify(g, fx["source"], dist) == 0


def test_fig1_unordered_worklist_revisits_A():
    """P:79 (§3.1): a FIFO (unordered) worklist that pops A before B processes A twice,
    the priority order processes each vertex once.  Pins the work counter semantics."""
    fx = load_golden("fig1_reconstructed.txt")
    n, s = fx["n"], fx["source"]
    adj = collections.defaultdict(list)
    for u, v, w in fx["arcs"]:
        adj[u].append((v, w))          # S's arcs in order (A, B)
    d = [INF] * n
    d[s] = 0
    q = collections.deque([s])
    processed = 0
    while q:
        u = q.popleft()
        processed += 1
        for v, w in adj[u]:
            if d[u] + w < d[v]:
                d[v] = d[u] + w
                q.append(v)
    assert d == fx["dist"]
    assert processed == 4            # S, A, B, A  (A visited twice)
    _, V, _ = oracle.dijkstra(gg.from_arcs(n, fx["arcs"]), s)
    assert V == 3                    # each vertex once


# ------------------------------------------------------------ brute force pins
@settings(max_examples=300, deadline=None)
@given(arc_lists)
def test_matches_floyd_warshall_and_bellman_ford(case):
    n, arcs, s = case
    g = gg.from_arcs(n, arcs)
    dist, V, E = oracle.dijkstra(g, s)
    fw = floyd_warshall(n, arcs)[s]
    bf = bellman_ford(n, arcs, s)
    assert [int(x) for x in dist] == fw == bf
    # work counts: each reachable vertex expanded exactly once (strict-improvement pushes)
    reach = [v for v in range(n) if fw[v] != INF]
    assert V == len(reach)
    assert E == sum(int(g.row_offsets[v + 1] - g.row_offsets[v]) for v in reach)
    assert oracle.certify(g, s, dist) == 0


def test_all_sources_tiny_random():
    rng = random.Random(7)
    for _ in range(30):
        n = rng.randint(1, 40)
        arcs = [(rng.randrange(n), rng.randrange(n), rng.randint(0, 50)) for _ in range(rng.randint(0, 5 * n))]
        g = gg.from_arcs(n, arcs)
        fw = floyd_warshall(n, arcs)
        for s in range(n):
            assert [int(x) for x in oracle.dijkstra(g, s)[0]] == fw[s]


# ------------------------------------------------------------ closed forms
def test_unit_weights_equal_bfs_hops():
    g = gg.rmat(12, 8, 1, 1, seed=11)
    for s in gg.sources(g, 3, seed=1):
        dist, _, _ = oracle.dijkstra(g, int(s))
        assert [int(x) for x in dist] == bfs_hops(g, int(s))


@pytest.mark.parametrize("c", [1, 7, 1000])
def test_constant_weight_is_c_times_hops(c):
    g = gg.er(3000, 12000, c, c, seed=5)
    hops = bfs_hops(g, 0)
    dist, _, _ = oracle.dijkstra(g, 0)
    assert [int(x) for x in dist] == [h if h == INF else c * h for h in hops]


@pytest.mark.parametrize("W,H,s", [(64, 64, 0), (50, 31, 777), (1, 9, 4), (17, 1, 16)])
def test_unit_grid_manhattan(W, H, s):
    g = gg.grid(W, H, 1, 1, seed=3)
    dist, V, E = oracle.dijkstra(g, s)
    sr, sc = divmod(s, W)
    want = [abs(v // W - sr) + abs(v % W - sc) for v in range(W * H)]
    assert [int(x) for x in dist] == want
    assert V == W * H and E == g.m


def test_path_graph_prefix_sums():
    rng = random.Random(3)
    n = 500
    ws = [rng.randint(0, 1 << 31) for _ in range(n - 1)]
    g = gg.from_arcs(n, [(i, i + 1, ws[i]) for i in range(n - 1)])
    dist, _, _ = oracle.dijkstra(g, 0)
    pref = [0]
    for x in ws:
        pref.append(pref[-1] + x)
    assert [int(x) for x in dist] == pref
    dist, _, _ = oracle.dijkstra(g, 100)
    assert [int(x) for x in dist] == [INF] * 100 + [p - pref[100] for p in pref[100:]]


def test_complete_dag():
    """w(i,j) = j - i for i < j  =>  dist[v] = v - s for v >= s, unreachable below s."""
    n = 60
    g = gg.from_arcs(n, [(i, j, j - i) for i in range(n) for j in range(i + 1, n)])
    for s in (0, 17, 59):
        dist, _, _ = oracle.dijkstra(g, s)
        assert [int(x) for x in dist] == [INF] * s + list(range(0, n - s))


def test_u32_overflow_needs_64bit_sums():
    n = 40
    g = gg.from_arcs(n, [(i, i + 1, 0xFFFFFFFF) for i in range(n - 1)])
    dist, _, _ = oracle.dijkstra(g, 0)
    assert [int(x) for x in dist] == [i * 0xFFFFFFFF for i in range(n)]


# ------------------------------------------------------------ library routine
def _scipy_dist(g, s):
    import scipy.sparse as sp
    from scipy.sparse.csgraph import dijkstra as sdij
    src = np.repeat(np.arange(g.n), np.diff(g.row_offsets).astype(np.int64))
    dst = g.col.astype(np.int64)
    w = g.w.astype(np.float64)
    # scipy's coo->csr SUMS duplicates, so min-reduce parallel arcs first
    order = np.lexsort((w, dst, src))
    src, dst, w = src[order], dst[order], w[order]
    keep = np.ones(len(src), bool)
    keep[1:] = (src[1:] != src[:-1]) | (dst[1:] != dst[:-1])
    src, dst, w = src[keep], dst[keep], w[keep]
    # scipy treats explicit zeros as "no edge": add a tiny epsilon and round back
    eps = 1.0 / (1 << 20)
    M = sp.csr_matrix((w + eps, (src, dst)), shape=(g.n, g.n))
    d = sdij(M, directed=True, indices=s)
    return d


@pytest.mark.parametrize("maker", [
    lambda: gg.rmat(13, 16, 1, 255, seed=3),
    lambda: gg.er(1 << 13, 32 << 13, 1, 1 << 20, seed=4),
    lambda: gg.make("grid64"),
    lambda: gg.grid(100, 80, 1, 1000, seed=9),
    lambda: gg.rmat(11, 8, 0, 3, seed=8),     # zero weights + many ties
])
def test_matches_scipy(maker):
    g = maker()
    for s in list(gg.sources(g, 2, seed=2)) + [0]:
        s = int(s)
        dist, _, _ = oracle.dijkstra(g, s)
        ref = _scipy_dist(g, s)
        fin = np.isfinite(ref)
        assert np.array_equal(dist != np.uint64(INF), fin)
        # the epsilon adds < (hops * 2^-20) < 0.5; rounding down recovers the exact integer sum
        assert np.array_equal(dist[fin], np.floor(ref[fin]).astype(np.uint64))


# ------------------------------------------------------------ certificate
def test_certificate_accepts_and_rejects():
    rng = np.random.default_rng(0)
    for g in (gg.rmat(12, 16, 1, 255, seed=3), gg.grid(40, 40, 1, 100, seed=1),
              gg.rmat(11, 8, 0, 2, seed=5)):
        s = int(gg.sources(g, 1, seed=1)[0])
        dist, _, _ = oracle.dijkstra(g, s)
        assert oracle.certify(g, s, dist) == 0
        fin = np.flatnonzero((dist != np.uint64(INF)) & (np.arange(g.n) != s))
        inf = np.flatnonzero(dist == np.uint64(INF))
        for v in rng.choice(fin, 20):
            for delta in (+1, -1):
                d2 = dist.copy()
                d2[v] = np.uint64(int(d2[v]) + delta)
                assert oracle.certify(g, s, d2) != 0, (v, delta)
            d2 = dist.copy()
            d2[v] = np.uint64(INF)           # finite -> infinite
            assert oracle.certify(g, s, d2) != 0
        for v in inf[:20]:
            d2 = dist.copy()
            d2[v] = np.uint64(5)             # infinite -> finite
            assert oracle.certify(g, s, d2) != 0
        d2 = dist.copy()
        d2[s] = np.uint64(1)
        assert oracle.certify(g, s, d2) != 0


def test_reach_counts_closed_form():
    g = gg.rmat(12, 16, 1, 255, seed=3)
    s = int(gg.sources(g, 1, seed=4)[0])
    dist, V, E = oracle.dijkstra(g, s)
    fin = dist != np.uint64(INF)
    deg = np.diff(g.row_offsets)
    assert V == int(fin.sum()) and E == int(deg[fin].sum())
    assert oracle.reach_counts(g, dist) == (V, E)

"""Pins for the float32-weight oracle (NEXT-3; the paper's float variant P:264).

Semantics (R16): dist[v] = min over paths of the IEEE binary32,
round-to-nearest, left-to-right path sum; +inf when unreachable.  Pins:
brute-force Bellman-Ford in numpy float32; dyadic weights whose sums are exact
reduce to the integer oracle; a hand-worked fixture where rounding decides."""
import random

import numpy as np
import pytest

import graphgen as gg
import oracle

F32 = np.float32


def bellman_ford_f32(n, arcs, s):
    d = [F32(np.inf)] * n
    d[s] = F32(0)
    for _ in range(max(n - 1, 1)):
        ch = False
        for u, v, w in arcs:
            nd = F32(d[u] + F32(w))          # binary32 RN addition
            if nd < d[v]:
                d[v] = nd
                ch = True
        if not ch:
            break
    return np.array(d, dtype=F32)


def _graph(n, arcs):
    g = gg.from_arcs(n, [(u, v, 0) for u, v, _ in arcs])
    # from_arcs sorts arcs by (u, v, w): rebuild the float weights in that order
    order = sorted(range(len(arcs)), key=lambda i: (arcs[i][0], arcs[i][1], 0, i))
    wf = np.array([arcs[i][2] for i in order], dtype=F32)
    return g, wf


@pytest.mark.parametrize("seed", range(40))
def test_matches_float32_bellman_ford(seed):
    rng = random.Random(seed)
    n = rng.randint(1, 40)
    arcs = [(rng.randrange(n), rng.randrange(n), F32(rng.choice([rng.random(), rng.random() * 1e-6,
                                                                 rng.random() * 1e6, 0.0])))
            for _ in range(rng.randint(0, 6 * n))]
    g, wf = _graph(n, arcs)
    s = rng.randrange(n)
    d, V, E = oracle.dijkstra_f32(g, wf, s)
    bf = bellman_ford_f32(n, [(u, v, w) for (u, v), w in zip(
        [(int(a), int(b)) for a, b in zip(np.repeat(np.arange(g.n), np.diff(g.row_offsets).astype(np.int64)), g.col)],
        wf)], s)
    assert np.array_equal(d.view(np.uint32), bf.view(np.uint32))


def test_dyadic_weights_are_exact():
    """weights k/8 with small sums are exact in binary32: float distances = int / 8."""
    g = gg.rmat(11, 8, 1, 64, seed=3)
    wf = (g.w.astype(np.float64) / 8.0).astype(F32)
    s = int(gg.sources(g, 1, seed=2)[0])
    di, V1, E1 = oracle.dijkstra(g, s)
    df, V2, E2 = oracle.dijkstra_f32(g, wf, s)
    fin = di != np.uint64(0xFFFFFFFFFFFFFFFF)
    assert np.array_equal(np.isfinite(df), fin)
    assert np.array_equal(df[fin].astype(np.float64) * 8.0, di[fin].astype(np.float64))
    assert (V1, E1) == (V2, E2)


def test_rounding_decides_hand_worked():
    """S->A 1.0, A->B 2^-24, S->B nextafter(1.0): exactly, S-A-B = 1 + 2^-24 is shorter
    than 1 + 2^-23, but in binary32 1.0 + 2^-24 rounds (ties-to-even) to 1.0, which is
    what the float variant computes (P:264 'handles floating point weights in the same way')."""
    one_ulp = np.nextafter(F32(1.0), F32(2.0))
    arcs = [(0, 1, F32(1.0)), (1, 2, F32(2.0 ** -24)), (0, 2, one_ulp)]
    g, wf = _graph(3, arcs)
    d, _, _ = oracle.dijkstra_f32(g, wf, 0)
    assert d[1] == F32(1.0)
    assert d[2] == F32(1.0) and d[2] < one_ulp


def test_unreachable_is_inf_and_zero_weights():
    g, wf = _graph(4, [(0, 1, F32(0.0)), (1, 2, F32(0.0)), (3, 0, F32(1.0))])
    d, V, E = oracle.dijkstra_f32(g, wf, 0)
    assert d[:3].tolist() == [0.0, 0.0, 0.0] and np.isinf(d[3])
    assert V == 3 and E == 2

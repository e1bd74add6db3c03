"""Loaders for the paper's input formats (NEXT-4): Galois binary .gr, DIMACS .gr,
MatrixMarket .mtx -- round trips and hand-written fixtures."""
import numpy as np
import pytest

import graphgen as gg
import oracle
from graphgen import loaders


def _same(a, b):
    return (a.n == b.n and a.m == b.m and np.array_equal(a.row_offsets, b.row_offsets)
            and np.array_equal(a.col, b.col) and np.array_equal(a.w, b.w))


@pytest.mark.parametrize("fmt", ["galois", "dimacs", "mtx"])
def test_round_trip(tmp_path, fmt):
    g = gg.rmat(9, 8, 1, 255, seed=3)
    p = str(tmp_path / f"g.{fmt}")
    {"galois": loaders.save_galois_gr, "dimacs": loaders.save_dimacs_gr, "mtx": loaders.save_mtx}[fmt](g, p)
    h = loaders.load(p)
    assert _same(g, h)
    s = int(gg.sources(g, 1, seed=1)[0])
    assert np.array_equal(oracle.dijkstra(g, s)[0], oracle.dijkstra(h, s)[0])


def test_odd_arc_count_padding(tmp_path):
    g = gg.from_arcs(3, [(0, 1, 5), (1, 2, 7), (2, 0, 1)])
    p = str(tmp_path / "odd.gr")
    loaders.save_galois_gr(g, p)
    assert _same(g, loaders.load_galois_gr(p))


def test_dimacs_fixture(tmp_path):
    p = tmp_path / "t.gr"
    p.write_text("c DIMACS 9th challenge format (P:522)\np sp 4 5\na 1 2 3\na 2 3 4\na 1 3 9\na 3 4 1\na 4 1 2\n")
    g = loaders.load(str(p))
    assert g.n == 4 and g.m == 5
    assert oracle.dijkstra(g, 0)[0].tolist() == [0, 3, 7, 8]


def test_mtx_symmetric_pattern_and_negative(tmp_path):
    p = tmp_path / "s.mtx"
    p.write_text("%%MatrixMarket matrix coordinate real symmetric\n% comment\n3 3 3\n2 1 -4.4\n3 2 2.6\n3 3 1.0\n")
    g = loaders.load(str(p))
    # symmetric expansion (diagonal kept once), |negative|, real rounded
    arcs = sorted(zip(np.repeat(np.arange(g.n), np.diff(g.row_offsets).astype(np.int64)).tolist(),
                      g.col.tolist(), g.w.tolist()))
    assert arcs == [(0, 1, 4), (1, 0, 4), (1, 2, 3), (2, 1, 3), (2, 2, 1)]
    q = tmp_path / "p.mtx"
    q.write_text("%%MatrixMarket matrix coordinate pattern general\n2 2 1\n1 2\n")
    h = loaders.load(str(q))
    assert h.m == 1 and h.w.tolist() == [1]


def test_bad_files(tmp_path):
    p = tmp_path / "bad.gr"
    p.write_text("c no header\na 1 2 3\n")
    with pytest.raises(ValueError):
        loaders.load_dimacs_gr(str(p))
    q = tmp_path / "bad.mtx"
    q.write_text("%%MatrixMarket matrix array real general\n2 2\n1\n2\n3\n4\n")
    with pytest.raises(ValueError):
        loaders.load_mtx(str(q))

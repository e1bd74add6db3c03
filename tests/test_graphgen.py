"""Generator tests: exact sizes, degree structure, ranges,
RMAT quadrant statistics, ER degree statistics, determinism across thread counts."""
import os
import subprocess
import sys

import numpy as np
import pytest

import graphgen as gg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _csr_ok(g):
    off = g.row_offsets
    assert off[0] == 0 and int(off[-1]) == g.m and len(off) == g.n + 1
    assert np.all(np.diff(off.astype(np.int64)) >= 0)
    assert g.col.size == g.m and g.w.size == g.m
    if g.m:
        assert int(g.col.max()) < g.n


@pytest.mark.parametrize("W,H", [(64, 64), (7, 5), (1, 3), (256, 128)])
def test_grid_structure(W, H):
    g = gg.grid(W, H, 1, 100, seed=1)
    _csr_ok(g)
    assert g.n == W * H and g.m == 2 * H * (W - 1) + 2 * W * (H - 1)
    deg = np.diff(g.row_offsets)
    if W >= 2 and H >= 2:
        hist = np.bincount(deg, minlength=5)
        assert hist[2] == 4
        assert hist[3] == 2 * (W - 2) + 2 * (H - 2)
        assert hist[4] == (W - 2) * (H - 2)
    # every arc joins lattice neighbours
    src = np.repeat(np.arange(g.n), deg.astype(np.int64))
    dr = np.abs(src // W - g.col // W)
    dc = np.abs(src % W - g.col % W)
    assert np.all(dr + dc == 1)
    assert g.w.min() >= 1 and g.w.max() <= 100


def test_config_sizes():
    g = gg.make("grid64")
    assert (g.n, g.m) == (4096, 16128)
    # ROAD at full size is cheap to build (closed-form lattice)
    r = gg.make("road")
    assert (r.n, r.m) == (16_777_216, 67_092_480)
    assert r.w.min() >= 1 and r.w.max() <= 1000
    # arcs u->v and v->u carry independent weights (A20)
    assert not np.array_equal(r.w[:1000], r.w[1000:2000])


def test_weights_uniform_inclusive_range():
    g = gg.er(1 << 14, 1 << 20, 3, 6, seed=2)
    cnt = np.bincount(g.w, minlength=8)[3:7]
    assert g.w.min() == 3 and g.w.max() == 6
    assert np.all(np.abs(cnt / g.m - 0.25) < 0.01)


def test_rmat_quadrant_frequencies():
    """Per-level (src bit, dst bit) frequencies match Graph500 (a,b,c,d) (chi-square)."""
    scale, ef = 14, 16
    g = gg.rmat(scale, ef, 1, 255, seed=3, permute=False)
    _csr_ok(g)
    assert g.n == 1 << scale and g.m == ef << scale
    src = np.repeat(np.arange(g.n, dtype=np.int64), np.diff(g.row_offsets).astype(np.int64))
    dst = g.col.astype(np.int64)
    p = np.array([37356, 12452, 12452, 65536 - 37356 - 2 * 12452]) / 65536.0
    for lvl in range(scale):
        q = ((src >> lvl) & 1) * 2 + ((dst >> lvl) & 1)
        obs = np.bincount(q, minlength=4)
        exp = p * g.m
        chi2 = float(((obs - exp) ** 2 / exp).sum())
        assert chi2 < 25.0, (lvl, obs, exp, chi2)     # 3 dof; p ~ 1.6e-5


def test_rmat_structure_scale16():
    g = gg.rmat(16, 16, 1, 255, seed=3)
    _csr_ok(g)
    deg = np.diff(g.row_offsets)
    assert 0.33 < (deg == 0).mean() < 0.45       # 0.383 at scale 16
    assert deg.max() > 5000
    assert g.w.min() >= 1 and g.w.max() <= 255


def test_er_degree_statistics():
    n = 1 << 16
    g = gg.er(n, 32 * n, 1, 1 << 20, seed=4)
    _csr_ok(g)
    deg = np.diff(g.row_offsets).astype(np.float64)
    assert deg.mean() == 32.0
    assert abs(deg.var() - 32.0) < 1.5                 # Poisson(32)
    indeg = np.bincount(g.col, minlength=n)
    assert abs(indeg.var() - 32.0) < 1.5


def test_rows_sorted_and_deterministic():
    g1 = gg.rmat(12, 16, 1, 255, seed=3)
    g2 = gg.rmat(12, 16, 1, 255, seed=3)
    assert g1.fingerprint() == g2.fingerprint()
    g3 = gg.rmat(12, 16, 1, 255, seed=4)
    assert g1.fingerprint() != g3.fingerprint()
    for v in range(0, g1.n, 97):
        b, e = int(g1.row_offsets[v]), int(g1.row_offsets[v + 1])
        key = g1.col[b:e].astype(np.uint64) << np.uint64(32) | g1.w[b:e]
        assert np.all(np.diff(key.astype(np.int64)) >= 0)


def test_fingerprint_independent_of_thread_count():
    code = ("import sys; sys.path.insert(0, %r); import graphgen as gg;"
            "print(gg.rmat(13,16,1,255,3).fingerprint(), gg.er(1<<13,32<<13,1,1<<20,4).fingerprint(),"
            " gg.make('grid64').fingerprint())" % ROOT)
    outs = []
    for t in ("1", "3", "8"):
        env = dict(os.environ, OMP_NUM_THREADS=t)
        outs.append(subprocess.check_output([sys.executable, "-c", code], env=env).strip())
    assert outs[0] == outs[1] == outs[2]


def test_sources_distinct_and_nonsink():
    g = gg.rmat(14, 16, 1, 255, seed=3)
    s = gg.sources(g, 512, seed=5)
    assert len(s) == 512 and len(set(s.tolist())) == 512
    deg = np.diff(g.row_offsets)
    assert np.all(deg[s] >= 1)
    assert np.array_equal(s, gg.sources(g, 512, seed=5))

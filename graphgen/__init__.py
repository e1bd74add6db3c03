"""Seeded synthetic CSR generators (inputs only -- no SSSP arithmetic here).

Shared by the oracle (``oracle/``) and the CUDA path; neither imports the
other.  The C implementation (``graphgen.c``) is compiled on first use with
gcc/OpenMP into ``graphgen/libgraphgen.so``.

Workloads (BASELINE.json ``configs``; recipe in DESIGN.md):

=========  =========================================================  =======
name       construction                                                seed
=========  =========================================================  =======
grid64     64x64 lattice, U[1,100], source 0                           1
road       4096x4096 lattice, U[1,1000], seeded source                 2
rmat       RMAT scale 24, edge factor 16, Graph500 abcd, U[1,255]      3
er         directed G(2^24, 32*2^24), U[1,2^20]                        4
batch      the ``rmat`` graph, 512 seeded distinct sources             3 / 5
=========  =========================================================  =======
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "graphgen.c")
_LIB = os.path.join(_HERE, "libgraphgen.so")
_lib = None

# Graph500 RMAT probabilities in 1/65536 units (0.57, 0.19, 0.19, 0.05 rounded)
RMAT_ABC = (37356, 12452, 12452)


def build(force: bool = False) -> str:
    """Compile graphgen.c -> libgraphgen.so (gcc -O3 -fopenmp)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        u64, u32, p = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p
        lib.gg_grid_arcs.restype = u64
        lib.gg_grid_arcs.argtypes = [u32, u32]
        lib.gg_grid.restype = ctypes.c_int
        lib.gg_grid.argtypes = [u32, u32, u32, u32, u64, p, p, p]
        lib.gg_rmat.restype = ctypes.c_int
        lib.gg_rmat.argtypes = [u32, u32, u32, u32, u32, u32, u32, u64, ctypes.c_int, p, p, p]
        lib.gg_er.restype = ctypes.c_int
        lib.gg_er.argtypes = [u64, u64, u32, u32, u64, p, p, p]
        lib.gg_sources.restype = u32
        lib.gg_sources.argtypes = [u64, p, u64, u32, p, u64]
        lib.gg_fingerprint.restype = u64
        lib.gg_fingerprint.argtypes = [u64, u64, p, p, p]
        lib.gg_hash.restype = u64
        lib.gg_hash.argtypes = [u64, u64, u64]
        lib.gg_num_threads.restype = ctypes.c_int
        lib.gg_float_weights.restype = None
        lib.gg_float_weights.argtypes = [u64, ctypes.c_float, ctypes.c_float, u64, p]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


@dataclass
class CSR:
    """Directed graph in CSR form: row_offsets uint64[n+1], col uint32[m], w uint32[m]."""
    n: int
    m: int
    row_offsets: np.ndarray
    col: np.ndarray
    w: np.ndarray
    name: str = "custom"
    seed: int = 0
    meta: dict = field(default_factory=dict)

    def fingerprint(self) -> int:
        return int(_L().gg_fingerprint(self.n, self.m, _ptr(self.row_offsets), _ptr(self.col), _ptr(self.w)))

    def out_degree(self) -> np.ndarray:
        return np.diff(self.row_offsets)

    def nbytes(self) -> int:
        return self.row_offsets.nbytes + self.col.nbytes + self.w.nbytes


def _alloc(n: int, m: int):
    return (np.empty(n + 1, dtype=np.uint64), np.empty(max(m, 1), dtype=np.uint32)[:m],
            np.empty(max(m, 1), dtype=np.uint32)[:m])


def grid(W: int, H: int, lo: int, hi: int, seed: int, name: str = "grid") -> CSR:
    """W x H 4-neighbour lattice, row-major ids, iid U[lo,hi] weight per directed arc."""
    lib = _L()
    n, m = W * H, int(lib.gg_grid_arcs(W, H))
    off, col, w = _alloc(n, m)
    rc = lib.gg_grid(W, H, lo, hi, seed, _ptr(off), _ptr(col), _ptr(w))
    assert rc == 0
    return CSR(n, m, off, col, w, name, seed, {"W": W, "H": H, "lo": lo, "hi": hi})


def rmat(scale: int, edge_factor: int, lo: int, hi: int, seed: int, name: str = "rmat",
         abc=RMAT_ABC, permute: bool = True) -> CSR:
    """Graph500 Kronecker graph, directed, duplicates/self-loops kept, permuted ids."""
    lib = _L()
    n, m = 1 << scale, edge_factor << scale
    off, col, w = _alloc(n, m)
    rc = lib.gg_rmat(scale, edge_factor, abc[0], abc[1], abc[2], lo, hi, seed, int(permute),
                     _ptr(off), _ptr(col), _ptr(w))
    if rc != 0:
        raise MemoryError("gg_rmat failed")
    return CSR(n, m, off, col, w, name, seed, {"scale": scale, "edge_factor": edge_factor, "lo": lo, "hi": hi})


def er(n: int, m: int, lo: int, hi: int, seed: int, name: str = "er") -> CSR:
    """Directed G(n, m): m arcs with iid uniform endpoints (duplicates/self-loops kept)."""
    lib = _L()
    off, col, w = _alloc(n, m)
    rc = lib.gg_er(n, m, lo, hi, seed, _ptr(off), _ptr(col), _ptr(w))
    if rc != 0:
        raise MemoryError("gg_er failed")
    return CSR(n, m, off, col, w, name, seed, {"lo": lo, "hi": hi})


def from_arcs(n: int, arcs, name: str = "custom") -> CSR:
    """Small helper for hand-made graphs: arcs = [(u, v, w), ...]; rows keep (v, w) order sorted."""
    arcs = sorted((int(u), int(v), int(w)) for u, v, w in arcs)
    m = len(arcs)
    off = np.zeros(n + 1, dtype=np.uint64)
    for u, _, _ in arcs:
        off[u + 1] += 1
    off = np.cumsum(off, dtype=np.uint64)
    col = np.array([a[1] for a in arcs], dtype=np.uint32)
    w = np.array([a[2] for a in arcs], dtype=np.uint32)
    return CSR(n, m, off, col, w, name, 0)


def sources(g: CSR, k: int, seed: int) -> np.ndarray:
    """First k distinct seeded draws among vertices with out-degree >= 1."""
    out = np.empty(max(k, 1), dtype=np.uint32)
    got = _L().gg_sources(g.n, _ptr(g.row_offsets), seed, k, _ptr(out), (1 << 20) + 64 * k)
    return out[:got].copy()


def float_weights(g: CSR, lo: float, hi: float, seed: int) -> np.ndarray:
    """float32 arc weights in [lo, hi) for graph g (NEXT-3), seeded and thread-count independent."""
    w = np.empty(max(g.m, 1), dtype=np.float32)[:g.m]
    _L().gg_float_weights(g.m, lo, hi, seed, _ptr(w))
    return w


def gg_hash(seed: int, stream: int, i: int) -> int:
    return int(_L().gg_hash(seed, stream, i))


def num_threads() -> int:
    return int(_L().gg_num_threads())


# --------------------------------------------------------------- configs
CONFIGS = {
    "grid64": dict(kind="grid", W=64, H=64, lo=1, hi=100, seed=1, source=0),
    "road": dict(kind="grid", W=4096, H=4096, lo=1, hi=1000, seed=2, source_seed=2),
    "rmat": dict(kind="rmat", scale=24, edge_factor=16, lo=1, hi=255, seed=3, source_seed=3),
    "er": dict(kind="er", n=1 << 24, m=32 << 24, lo=1, hi=1 << 20, seed=4, source_seed=4),
    "batch": dict(kind="rmat", scale=24, edge_factor=16, lo=1, hi=255, seed=3, source_seed=5, k=512),
}
# Further families (not BASELINE configs): controller / launch-default validation on graphs
# that sit on the other side of the defaults' average-degree switch (<= 8 arcs per vertex
# selects the latency build) or change the weight range by orders of magnitude.
EXTRA = {
    "rmat_ef4": dict(kind="rmat", scale=24, edge_factor=4, lo=1, hi=255, seed=6, source_seed=6),
    "er_d4": dict(kind="er", n=1 << 24, m=4 << 24, lo=1, hi=1 << 20, seed=7, source_seed=7),
    "grid_wide": dict(kind="grid", W=4096, H=4096, lo=1, hi=1 << 20, seed=8, source_seed=8),
    "rmat_wide": dict(kind="rmat", scale=24, edge_factor=16, lo=1, hi=1 << 20, seed=9, source_seed=9),
}


def make(config: str, scale_down: int = 0) -> CSR:
    """Build a named config graph.  ``scale_down`` shrinks it by 2^scale_down
    vertices (same recipe) for tests that must stay small."""
    c = CONFIGS[config] if config in CONFIGS else EXTRA[config]
    if c["kind"] == "grid":
        W = max(2, c["W"] >> (scale_down // 2 + scale_down % 2))
        H = max(2, c["H"] >> (scale_down // 2))
        return grid(W, H, c["lo"], c["hi"], c["seed"], name=config)
    if c["kind"] == "rmat":
        return rmat(c["scale"] - scale_down, c["edge_factor"], c["lo"], c["hi"], c["seed"], name=config)
    if c["kind"] == "er":
        n = c["n"] >> scale_down
        return er(n, c["m"] >> scale_down, c["lo"], c["hi"], c["seed"], name=config)
    raise KeyError(config)


def config_sources(config: str, g: CSR, k: int = 1) -> np.ndarray:
    c = CONFIGS[config] if config in CONFIGS else EXTRA[config]
    if "source" in c:
        return np.array([c["source"]] * k, dtype=np.uint32)[:k]
    return sources(g, k, c["source_seed"])

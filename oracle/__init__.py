"""CPU oracle for the ADDS SSSP hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_ppopp_wangfl21_b200``) must never import it; it
shares no code with the CUDA path (see ``oracle.c`` header for the paper
passages each function follows).

Functions
---------
dijkstra(g, s)        -> (dist uint64[n], V_dij, E_dij)   binary-heap Dijkstra
dijkstra_f32(g, wf, s)-> float32 distances with IEEE-rounded path sums (NEXT-3)
certify(g, s, dist)   -> 0 if dist is exact, else clause code
reach_counts(g, dist) -> (V, E) recomputed from a distance vector
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

INF = np.uint64(0xFFFFFFFFFFFFFFFF)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (plain gcc -O2, single thread)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        u64, u32, p = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p
        lib.oracle_dijkstra.restype = ctypes.c_int
        lib.oracle_dijkstra.argtypes = [u64, u64, p, p, p, u32, p, p, p]
        lib.oracle_certify.restype = ctypes.c_int
        lib.oracle_certify.argtypes = [u64, u64, p, p, p, u32, p, p]
        lib.oracle_dijkstra_f32.restype = ctypes.c_int
        lib.oracle_dijkstra_f32.argtypes = [u64, u64, p, p, p, u32, p, p, p]
        lib.oracle_reach_counts.restype = None
        lib.oracle_reach_counts.argtypes = [u64, p, p, p, p]
        _lib = lib
    return _lib


def _arrays(g):
    off = np.ascontiguousarray(g.row_offsets, dtype=np.uint64)
    col = np.ascontiguousarray(g.col, dtype=np.uint32)
    w = np.ascontiguousarray(g.w, dtype=np.uint32)
    return off, col, w


def dijkstra(g, s: int):
    """Exact SSSP distances from ``s`` (uint64, unreachable = 2^64-1) and work counts."""
    off, col, w = _arrays(g)
    n = len(off) - 1
    dist = np.empty(n, dtype=np.uint64)
    V = ctypes.c_uint64(0)
    E = ctypes.c_uint64(0)
    rc = _L().oracle_dijkstra(n, len(col), off.ctypes.data, col.ctypes.data, w.ctypes.data, int(s),
                              dist.ctypes.data, ctypes.byref(V), ctypes.byref(E))
    if rc != 0:
        raise ValueError(f"oracle_dijkstra failed (rc={rc})")
    return dist, int(V.value), int(E.value)


def dijkstra_f32(g, wf, s: int):
    """Float32-weight SSSP (NEXT-3): dist[v] = min over paths of the float-rounded
    left-to-right path sum; +inf when unreachable.  ``wf`` = float32[m] weights."""
    off, col, _ = _arrays(g)
    w = np.ascontiguousarray(wf, dtype=np.float32)
    n = len(off) - 1
    dist = np.empty(n, dtype=np.float32)
    V = ctypes.c_uint64(0)
    E = ctypes.c_uint64(0)
    rc = _L().oracle_dijkstra_f32(n, len(col), off.ctypes.data, col.ctypes.data, w.ctypes.data, int(s),
                                  dist.ctypes.data, ctypes.byref(V), ctypes.byref(E))
    if rc != 0:
        raise ValueError(f"oracle_dijkstra_f32 failed (rc={rc})")
    return dist, int(V.value), int(E.value)


def certify(g, s: int, dist) -> int:
    """0 iff ``dist`` is the exact distance vector; 1/2/3 = violated clause."""
    off, col, w = _arrays(g)
    d = np.ascontiguousarray(dist, dtype=np.uint64)
    bad = ctypes.c_uint64(0)
    return int(_L().oracle_certify(len(off) - 1, len(col), off.ctypes.data, col.ctypes.data,
                                   w.ctypes.data, int(s), d.ctypes.data, ctypes.byref(bad)))


def reach_counts(g, dist):
    off, _, _ = _arrays(g)
    d = np.ascontiguousarray(dist, dtype=np.uint64)
    V = ctypes.c_uint64(0)
    E = ctypes.c_uint64(0)
    _L().oracle_reach_counts(len(off) - 1, off.ctypes.data, d.ctypes.data, ctypes.byref(V), ctypes.byref(E))
    return int(V.value), int(E.value)

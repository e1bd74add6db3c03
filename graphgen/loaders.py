"""Graph file loaders / writers (inputs only, no SSSP arithmetic).

The paper's inputs are Galois binary ``.gr`` files, converted from SuiteSparse
MatrixMarket files, plus the DIMACS-challenge road graphs (
the link at P:522 is the DIMACS 9th-challenge format page although the text
calls the file "binary" -- reading R24 in DESIGN.md: both formats are
supported).  Every loader returns a :class:`graphgen.CSR` with uint64 row
offsets, uint32 columns and uint32 weights, rows sorted by (col, w).

Conversions (recorded in ``CSR.meta``): negative weights are made positive as
the paper did; MatrixMarket ``real`` values are rounded to the nearest
integer, ``pattern`` matrices get weight 1, ``symmetric`` matrices are expanded
to both directions.
"""
from __future__ import annotations

import numpy as np

from . import CSR


def _to_csr(n, src, dst, w, name, meta) -> CSR:
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    w = np.asarray(w, dtype=np.uint64)
    if src.size and (src.min() < 0 or dst.min() < 0 or src.max() >= n or dst.max() >= n):
        raise ValueError("vertex id out of range")
    if w.size and w.max() > 0xFFFFFFFF:
        raise ValueError("weight exceeds uint32")
    order = np.lexsort((w, dst, src))
    src, dst, w = src[order], dst[order], w[order]
    off = np.zeros(n + 1, dtype=np.uint64)
    np.add.at(off, src + 1, 1)
    off = np.cumsum(off, dtype=np.uint64)
    return CSR(n, int(len(src)), off, dst.astype(np.uint32), w.astype(np.uint32), name, 0, meta)


# ------------------------------------------------------------------ Galois binary .gr (version 1)
# layout: u64 version=1, u64 sizeof(edge data), u64 n, u64 m, u64 out_end[n],
#         u32 dst[m], (u32 pad if m is odd), edge data[m]
def load_galois_gr(path: str, name: str | None = None) -> CSR:
    with open(path, "rb") as f:
        hdr = np.fromfile(f, dtype=np.uint64, count=4)
        if hdr.size != 4 or int(hdr[0]) != 1:
            raise ValueError(f"{path}: not a version-1 Galois .gr file")
        esz, n, m = int(hdr[1]), int(hdr[2]), int(hdr[3])
        ends = np.fromfile(f, dtype=np.uint64, count=n)
        dst = np.fromfile(f, dtype=np.uint32, count=m)
        if m % 2:
            np.fromfile(f, dtype=np.uint32, count=1)
        if esz == 4:
            w = np.fromfile(f, dtype=np.int32, count=m).astype(np.int64)
        elif esz == 0:
            w = np.ones(m, dtype=np.int64)
        else:
            raise ValueError(f"{path}: edge data of {esz} bytes not supported (uint32/int32 weights only)")
    if ends.size != n or dst.size != m or w.size != m:
        raise ValueError(f"{path}: truncated")
    off = np.concatenate([[0], ends]).astype(np.uint64)
    if np.any(np.diff(off.astype(np.int64)) < 0) or (n and int(off[-1]) != m):
        raise ValueError(f"{path}: inconsistent offsets")
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(off).astype(np.int64))
    neg = int((w < 0).sum())
    return _to_csr(n, src, dst, np.abs(w), name or path, {"format": "galois-gr", "negated_weights": neg})


def save_galois_gr(g: CSR, path: str) -> None:
    with open(path, "wb") as f:
        np.array([1, 4, g.n, g.m], dtype=np.uint64).tofile(f)
        g.row_offsets[1:].astype(np.uint64).tofile(f)
        g.col.astype(np.uint32).tofile(f)
        if g.m % 2:
            np.zeros(1, dtype=np.uint32).tofile(f)
        g.w.astype(np.uint32).tofile(f)


# ------------------------------------------------------------------ DIMACS 9th challenge .gr (text)
def load_dimacs_gr(path: str, name: str | None = None) -> CSR:
    n = m = None
    src, dst, w = [], [], []
    with open(path) as f:
        for line in f:
            if not line or line[0] == "c" or line[0] == "\n":
                continue
            t = line.split()
            if t[0] == "p":
                n, m = int(t[2]), int(t[3])
            elif t[0] == "a":
                src.append(int(t[1]) - 1)
                dst.append(int(t[2]) - 1)
                w.append(int(t[3]))
    if n is None:
        raise ValueError(f"{path}: missing 'p sp n m' line")
    if m is not None and m != len(src):
        raise ValueError(f"{path}: header says {m} arcs, found {len(src)}")
    w = np.abs(np.asarray(w, dtype=np.int64))
    return _to_csr(n, src, dst, w, name or path, {"format": "dimacs-gr"})


def save_dimacs_gr(g: CSR, path: str) -> None:
    src = np.repeat(np.arange(g.n), np.diff(g.row_offsets).astype(np.int64))
    with open(path, "w") as f:
        f.write(f"c written by graphgen.loaders\np sp {g.n} {g.m}\n")
        for u, v, ww in zip(src, g.col, g.w):
            f.write(f"a {u + 1} {int(v) + 1} {int(ww)}\n")


# ------------------------------------------------------------------ MatrixMarket coordinate .mtx
def load_mtx(path: str, name: str | None = None) -> CSR:
    with open(path) as f:
        banner = f.readline().lower().split()
        if len(banner) < 5 or banner[0] != "%%matrixmarket" or banner[2] != "coordinate":
            raise ValueError(f"{path}: only MatrixMarket coordinate matrices are supported")
        field, sym = banner[3], banner[4]
        line = f.readline()
        while line.startswith("%"):
            line = f.readline()
        rows, cols, nnz = (int(x) for x in line.split())
        data = np.loadtxt(f, ndmin=2) if nnz else np.zeros((0, 3))
    n = max(rows, cols)
    i = data[:, 0].astype(np.int64) - 1
    j = data[:, 1].astype(np.int64) - 1
    if field == "pattern":
        v = np.ones(len(i), dtype=np.int64)
    else:
        v = np.rint(np.abs(data[:, 2])).astype(np.int64)
    if sym in ("symmetric", "skew-symmetric", "hermitian"):
        off = i != j
        i, j, v = np.concatenate([i, j[off]]), np.concatenate([j, i[off]]), np.concatenate([v, v[off]])
    return _to_csr(n, i, j, v, name or path, {"format": "mtx", "field": field, "symmetry": sym})


def save_mtx(g: CSR, path: str) -> None:
    src = np.repeat(np.arange(g.n), np.diff(g.row_offsets).astype(np.int64))
    with open(path, "w") as f:
        f.write("%%MatrixMarket matrix coordinate integer general\n")
        f.write(f"{g.n} {g.n} {g.m}\n")
        for u, v, ww in zip(src, g.col, g.w):
            f.write(f"{u + 1} {int(v) + 1} {int(ww)}\n")


def load(path: str) -> CSR:
    """Dispatch on content: Galois binary .gr, DIMACS text .gr, or .mtx."""
    with open(path, "rb") as f:
        head = f.read(16)
    if head[:2] == b"%%":
        return load_mtx(path)
    if len(head) >= 8 and int(np.frombuffer(head[:8], dtype=np.uint64)[0]) == 1:
        return load_galois_gr(path)
    return load_dimacs_gr(path)

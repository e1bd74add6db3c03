#!/usr/bin/env python
"""Run the GPU SSSP on a graph file (Galois .gr, DIMACS .gr or .mtx; NEXT-4):

    python tools/run_file.py graph.gr [--source S] [--verify]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402
from graphgen import loaders  # noqa: E402
import paper_conf_ppopp_wangfl21_b200 as sssp  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("path")
    ap.add_argument("--source", type=int, default=None)
    ap.add_argument("--verify", action="store_true", help="compare with the CPU oracle (test infrastructure)")
    a = ap.parse_args()
    g = loaders.load(a.path)
    s = a.source if a.source is not None else int(gg.sources(g, 1, seed=1)[0])
    G = sssp.Graph.from_csr(g)
    d = sssp.to_u64(G.run(s))
    st = G.stats()
    out = {"n": g.n, "m": g.m, "source": s, "kernel_ms": st["kernel_ms"], "reachable": st["reachable"],
           "gteps": st["reach_edges"] / max(st["kernel_ms"], 1e-9) / 1e6,
           "work_edges": st["edges_relaxed"] / max(1, st["reach_edges"]), "max_dist": st["max_dist"]}
    if a.verify:
        import oracle
        out["bit_exact"] = bool(np.array_equal(d, oracle.dijkstra(g, s)[0]))
    print(json.dumps(out))


if __name__ == "__main__":
    main()

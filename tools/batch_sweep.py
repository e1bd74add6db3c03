#!/usr/bin/env python
"""Multi-source batch throughput vs sources in flight (NEXT-1, options.concurrent_sources).

For a config, k seeded sources run through sssp_run_batch at each concurrency c (one
warm-up batch, R timed batches, CUDA events on the stream); prints ms/source, GTEPS
(E_dij / time) and work per c.

    python tools/batch_sweep.py --config road --k 64 --conc 1,2,4,8 [--reps 2]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import graphgen as gg  # noqa: E402
import paper_conf_ppopp_wangfl21_b200 as sssp  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="road")
    ap.add_argument("--k", type=int, default=64)
    ap.add_argument("--conc", default="1,2,4,8")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--variant", default="")
    ap.add_argument("--opts", default="{}")
    a = ap.parse_args()
    import torch
    g = gg.make(a.config)
    srcs = gg.config_sources(a.config, g, a.k) if a.config != "batch" else gg.sources(
        g, a.k, gg.CONFIGS["batch"]["source_seed"])
    G = sssp.Graph.from_csr(g, variant=a.variant, **json.loads(a.opts))
    out = torch.empty((a.k, g.n), dtype=torch.int64, device="cuda")
    st = torch.cuda.current_stream()
    for c in [int(x) for x in a.conc.split(",")]:
        G.set_options(concurrent_sources=c)
        G.run_batch(srcs, out=out, stream=st)  # warm-up (allocates c workspaces)
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        torch.cuda.synchronize()
        ev[0].record(st)
        acc = dict(E=0, Eg=0, V=0, Vg=0)
        for _ in range(a.reps):
            G.run_batch(srcs, out=out, stream=st)
            s = G.stats()
            acc["E"] += s["reach_edges"]
            acc["Eg"] += s["edges_relaxed"]
        ev[1].record(st)
        torch.cuda.synchronize()
        ms = ev[0].elapsed_time(ev[1])
        print(json.dumps({"config": a.config, "k": a.k, "concurrent_sources": c,
                          "ms_per_source": round(ms / (a.reps * a.k), 3),
                          "gteps": round(acc["E"] / (ms / 1e3) / 1e9, 2),
                          "work_E": round(acc["Eg"] / max(1, acc["E"]), 3)}), flush=True)


if __name__ == "__main__":
    main()

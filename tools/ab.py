#!/usr/bin/env python
"""Interleaved A/B of library builds on the GPU box.

Each variant name V loads paper_conf_ppopp_wangfl21_b200/libsssp_V.so ("" = the
product libsssp.so).  For every config the graph is generated once and one
handle per variant is created on it; then, for R repetitions of S seeded
sources, the variants run the same source back to back (alternating order), so
box-to-box and thermal drift hit every variant alike.  Prints one JSON line per
(config, variant): median / min kernel ms, GTEPS, work efficiency.

    python tools/ab.py --variants ",base" --configs rmat,er --sources 4 --reps 2 [--opts '{...}']
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import graphgen as gg  # noqa: E402
import paper_conf_ppopp_wangfl21_b200 as sssp  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--variants", default=",base")
    ap.add_argument("--configs", default="rmat,er,road")
    ap.add_argument("--sources", type=int, default=4)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--scale-down", type=int, default=0)
    ap.add_argument("--opts", default="{}", help="JSON options for every variant")
    ap.add_argument("--vopts", default="{}", help="JSON {variant: options} overriding --opts per variant")
    a = ap.parse_args()
    import torch
    variants = a.variants.split(",")
    vopts = json.loads(a.vopts)
    for cfg in a.configs.split(","):
        g = gg.make(cfg, scale_down=a.scale_down)
        srcs = gg.config_sources(cfg, g, a.sources)
        Gs = {}
        for v in variants:
            o = dict(json.loads(a.opts))
            o.update(vopts.get(v, {}))
            lib_v = v.split(":")[0]
            Gs[v] = sssp.Graph.from_csr(g, variant=lib_v, **o)
        out = torch.empty(g.n, dtype=torch.int64, device="cuda")
        for v in variants:  # warm-up
            Gs[v].run(int(srcs[0]), out=out)
        res = {v: dict(ms=[], Eg=0, Ed=0, Vg=0, Vd=0, k=[]) for v in variants}
        ref = None
        for r in range(a.reps):
            for i, s in enumerate(srcs):
                order = variants if (r + i) % 2 == 0 else variants[::-1]
                for v in order:
                    Gs[v].run(int(s), out=out)
                    st = Gs[v].stats()
                    q = res[v]
                    q["ms"].append(st["kernel_ms"])
                    q["Eg"] += st["edges_relaxed"]
                    q["Ed"] += st["reach_edges"]
                    q["Vg"] += st["vertices_processed"]
                    q["Vd"] += st["reachable"]
                    q["k"].append(st["final_delta_log2"])
                    if r == 0 and i == 0:
                        h = out.cpu()
                        if ref is None:
                            ref = h
                        elif not torch.equal(ref, h):
                            print(json.dumps({"config": cfg, "variant": v, "error": "distances differ"}), flush=True)
        for v in variants:
            q = res[v]
            ms = statistics.median(q["ms"])
            print(json.dumps({"config": cfg, "variant": v or "(product)", "median_ms": round(ms, 3),
                              "min_ms": round(min(q["ms"]), 3), "gteps": round(q["Ed"] / len(q["ms"]) / ms / 1e6, 2),
                              "work_E": round(q["Eg"] / q["Ed"], 3), "work_V": round(q["Vg"] / q["Vd"], 3),
                              "final_k": sorted(set(q["k"]))}), flush=True)
        for v in variants:
            Gs[v].close()
        del Gs, out, g
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()

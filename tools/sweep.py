#!/usr/bin/env python
"""Static-Delta / launch-shape sweep (the Fig. 4/7 analog).

Runs on the GPU box: for each config, every option set, a few seeded sources;
prints one JSON line per (config, option set) with median kernel ms, GTEPS and
work efficiency (E_gpu/E_dij, V_gpu/V_dij)."""
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
    ap.add_argument("--config", default="road")
    ap.add_argument("--scale-down", type=int, default=0)
    ap.add_argument("--sources", type=int, default=2)
    ap.add_argument("--sets", default="[]", help="JSON list of option dicts")
    ap.add_argument("--deltas", default="", help="comma list of log2 Delta for static sweeps")
    ap.add_argument("--extra", default="{}", help="JSON dict merged into every static set")
    ap.add_argument("--profile", action="store_true", help="add SSSP_FLAG_PROFILE and print phase fractions")
    ap.add_argument("--variant", default="", help="library build: loads libsssp_<variant>.so")
    a = ap.parse_args()
    import torch
    g = gg.make(a.config, scale_down=a.scale_down)
    srcs = gg.config_sources(a.config, g, a.sources)
    sets = json.loads(a.sets)
    extra = json.loads(a.extra)
    for k in [int(x) for x in a.deltas.split(",") if x]:
        sets.append(dict(delta_mode=1, delta_init=1 << k, **extra))
    G = sssp.Graph.from_csr(g, variant=a.variant)
    base = sssp.sssp_options_default()
    out = torch.empty(g.n, dtype=torch.int64, device="cuda")
    for s in sets:
        o = sssp.sssp_options_default()
        for kk, v in s.items():
            setattr(o, kk, v)
        if a.profile:
            o.flags |= sssp.SSSP_FLAG_PROFILE
        sssp._check(sssp.lib().sssp_set_options(G._h, o))
        G.options = o
        G.run(int(srcs[0]), out=out)  # warm
        ks, Eg, Ed, Vg, Vd, dl = [], 0, 0, 0, 0, []
        for src in srcs:
            G.run(int(src), out=out)
            st = G.stats()
            ks.append(st["kernel_ms"])
            Eg += st["edges_relaxed"]; Ed += st["reach_edges"]; Vg += st["vertices_processed"]; Vd += st["reachable"]
            dl.append(st["final_delta_log2"])
        ms = statistics.median(ks)
        prof = None
        if a.profile:
            pr = G.profile()
            tot = max(1, pr["cyc_total"])
            prof = {k[4:]: round(v / tot, 3) for k, v in pr.items() if k.startswith("cyc_") and k != "cyc_total"}
            prof.update({k: v for k, v in pr.items() if k.startswith("n_")})
            nb = max(1, pr["n_ring_batches"] + pr["n_local_batches"])
            prof["cyc_per_batch"] = round((pr["cyc_total"] - pr["cyc_idle"]) / nb, 1)
            prof["rounds_per_batch"] = round(pr["n_rounds"] / nb, 2)
            prof["items_per_batch"] = round((st["vertices_processed"] + st["stale_skips"]) / nb, 1)
        print(json.dumps({"prof": prof, "config": a.config, "opts": s, "kernel_ms": round(ms, 3),
                          "gteps": round(Ed / len(srcs) / ms / 1e6, 2), "work_E": round(Eg / Ed, 3),
                          "work_V": round(Vg / Vd, 3), "final_k": dl, "head_switches": st["head_switches"]}),
              flush=True)


if __name__ == "__main__":
    main()

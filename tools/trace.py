#!/usr/bin/env python
"""Delta-controller trace (Figs. 11-15 analog): run one source with
SSSP_FLAG_TRACE and print a sampled table of (time, head, Delta, active buckets,
pending items total/window/tail)."""
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
    ap.add_argument("--scale-down", type=int, default=0)
    ap.add_argument("--opts", default="{}")
    ap.add_argument("--rows", type=int, default=24)
    ap.add_argument("--variant", default="", help="library build: loads libsssp_<variant>.so")
    ap.add_argument("--changes", action="store_true", help="also print every entry where Delta or A changed")
    a = ap.parse_args()
    g = gg.make(a.config, scale_down=a.scale_down)
    s = int(gg.config_sources(a.config, g, 1)[0])
    opts = json.loads(a.opts)
    opts["flags"] = opts.get("flags", 0) | sssp.SSSP_FLAG_TRACE
    G = sssp.Graph.from_csr(g, variant=a.variant, **opts)
    G.run(s)
    G.run(s)
    st = G.stats()
    tr = G.trace()
    print(json.dumps({k: st[k] for k in ("kernel_ms", "init_delta_log2", "final_delta_log2", "head_switches",
                                         "delta_changes", "edges_relaxed", "reach_edges")}))
    if not tr:
        return
    t0 = tr[0]["time_ns"]
    step = max(1, len(tr) // a.rows)
    rows = tr[::step]
    if a.changes:
        keep = {0}
        for i in range(1, len(tr)):
            if (tr[i]["delta_log2"], tr[i]["active"] & 255) != (tr[i - 1]["delta_log2"], tr[i - 1]["active"] & 255):
                keep.update({i - 1, i})
        rows = [tr[i] for i in sorted(keep | set(range(0, len(tr), step)))]
    for e in rows:
        print(f'{(e["time_ns"] - t0) / 1e3:9.1f}us head={e["head"]:8d} k={e["delta_log2"]:2d} A={e["active"] & 255:2d} '
              f'flo={(e["active"] >> 8) & 255:2d} '
              f'pend={e["pending_total"]:9d} win={e["pending_window"]:9d} tail={e["pending_tail"]:8d} '
              f'waste={e["waste_permille"]:4d} clip={(e["reason"] >> 20) & 1023:4d}{"*" if e["reason"] >> 30 & 1 else " "} '
              f'why={e["reason"] & 255} flags={(e["reason"] >> 8) & 511:09b}')


if __name__ == "__main__":
    main()

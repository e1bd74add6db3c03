#!/usr/bin/env python
"""Hunt for timing-dependent controller spirals: run seeded sources of a config R times each
with the Delta trace on, print one line per run (kernel ms, work, initial/final Delta, Delta
changes) and the Delta/active-bucket changes of the run with the most work."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import graphgen as gg  # noqa: E402
import paper_conf_ppopp_wangfl21_b200 as sssp  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "road"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    trace = "notrace" not in sys.argv
    g = gg.make(cfg)
    srcs = gg.config_sources(cfg, g, 8)
    G = sssp.Graph.from_csr(g, flags=sssp.SSSP_FLAG_TRACE if trace else 0)
    worst = None
    for r in range(reps):
        for s in srcs:
            G.run(int(s))
            st = G.stats()
            w = st["edges_relaxed"] / max(1, st["reach_edges"])
            print(json.dumps({"rep": r, "src": int(s), "kernel_ms": round(st["kernel_ms"], 2), "work": round(w, 3),
                              "k0": st["init_delta_log2"], "k": st["final_delta_log2"],
                              "changes": st["delta_changes"], "switches": st["head_switches"]}), flush=True)
            if worst is None or w > worst[0]:
                worst = (w, int(s), G.trace() if trace else [])
    w, s, tr = worst
    if not tr:
        return
    print(f"# worst run: source {s}, work {w:.3f}; Delta / A changes:")
    t0 = tr[0]["time_ns"]
    for i in range(1, len(tr)):
        a, b = tr[i - 1], tr[i]
        if (a["delta_log2"], a["active"] & 255) != (b["delta_log2"], b["active"] & 255):
            print(f'{(b["time_ns"] - t0) / 1e3:9.1f}us head={b["head"]:8d} k={a["delta_log2"]}->{b["delta_log2"]} '
                  f'A={a["active"] & 255}->{b["active"] & 255} pend={b["pending_total"]} win={b["pending_window"]} '
                  f'tail={b["pending_tail"]} waste={b["waste_permille"]} why={b["reason"] & 255} '
                  f'flags={(b["reason"] >> 8) & 511:09b}')


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Small SSSP runs for compute-sanitizer (memcheck / synccheck / racecheck): grid64 and
scaled-down ROAD/RMAT/ER (2^-10), one source each through the C ABI, checked bit-exactly
against the CPU oracle (test infrastructure: this tool is run only on the GPU box).

    compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ppopp_wangfl21_b200 as sssp  # noqa: E402


def main():
    variant = sys.argv[1] if len(sys.argv) > 1 else ""
    cases = [("grid64", 0), ("road", 10), ("rmat", 10), ("er", 10)]
    for cfg, down in cases:
        g = gg.make(cfg, scale_down=down)
        s = int(gg.config_sources(cfg, g, 1)[0])
        G = sssp.Graph.from_csr(g, device=0, variant=variant)
        d = sssp.to_u64(G.run(s))
        ref, _, _ = oracle.dijkstra(g, s)
        assert np.array_equal(d, ref), cfg
        b = sssp.to_u64(G.run_batch(gg.config_sources(cfg, g, 2)).reshape(-1)).reshape(2, -1)
        assert np.array_equal(b[0], ref)
        G.close()
        print(f"{cfg} (scale_down {down}): n={g.n} m={g.m} exact", flush=True)


if __name__ == "__main__":
    main()

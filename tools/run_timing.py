#!/usr/bin/env python
"""Wall vs kernel time of single-source runs (one config, a few sources): sssp_run device time
around each call next to the kernel time the library reports, and the retry count."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import graphgen as gg  # noqa: E402
import paper_conf_ppopp_wangfl21_b200 as sssp  # noqa: E402


def main():
    import torch
    cfg = sys.argv[1] if len(sys.argv) > 1 else "road"
    variants = sys.argv[2].split(",") if len(sys.argv) > 2 else [""]
    g = gg.make(cfg)
    srcs = gg.config_sources(cfg, g, 6)
    out = torch.empty(g.n, dtype=torch.int64, device="cuda")
    st = torch.cuda.current_stream()
    for v in variants:
        G = sssp.Graph.from_csr(g, variant=v)
        for s in srcs:
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            ev[0].record(st)
            G.run(int(s), out=out, stream=st)
            ev[1].record(st)
            torch.cuda.synchronize()
            w = (time.perf_counter() - t0) * 1e3
            x = G.stats()
            print(f"{v or 'product'} src={int(s)} event_ms={ev[0].elapsed_time(ev[1]):.2f} wall_ms={w:.2f} "
                  f"kernel_ms={x['kernel_ms']:.2f} retries={x['retries']} ring_bytes={x['ring_bytes']}", flush=True)
        G.close()


if __name__ == "__main__":
    main()

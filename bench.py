#!/usr/bin/env python
"""Benchmark of the ADDS SSSP hot path on B200 (one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config batch|rmat|er|road|grid64]
                    [--impl ours|reference] [--no-singles]

Default workload = BASELINE.json configs[4] (config 5): RMAT scale 24, edge
factor 16, U[1,255], a batch of 512 seeded sources partitioned by source across
the ranks (``sources[rank::N]``), the CSR replicated on every GPU.  One step =
one pass over the batch: every rank runs its slice through
``distributed.run_batch_distributed`` (sssp_run_batch, several sources in flight
per GPU), the same rank loop the gloo tests drive.  The K timed steps are
bracketed by barrier + synchronize on both sides and timed with CUDA events on
the run stream; the max over ranks is taken.  ``value`` = GTEPS = (sum over
ranks and steps of E_dij, the arcs out of reachable vertices: Graph500-style
algorithmic TEPS, R2) / time.  The total work is fixed (512 sources),
so the scaling over N is strong scaling.

At N = 1 the line also carries ``singles``: the single-source configs 2-4 (ROAD,
RMAT-24 and ER-2^24, the largest single-GPU config), each with its own
ms/source, GTEPS, work efficiency, ``roofline`` and 1-core ``cpu_baseline``.

--impl reference times the CPU oracle (binary-heap Dijkstra, the paper's own
serial baseline P:268) on the same workload: a step is a bounded sample of the
batch, one source per host core on every core at once.  It is one of the three
places allowed to run oracle/.
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402

WORKLOADS = {
    "batch": "config 5: RMAT scale 24 edge factor 16 (Graph500 abcd), n=16,777,216 m=268,435,456, U[1,255], "
             "512 seeded sources partitioned by source across the GPUs, CSR replicated",
    "grid64": "config 1: 64x64 grid, 4-neighbour, U[1,100], source 0",
    "road": "config 2: 4096x4096 perturbed grid (road-like), n=16,777,216 m=67,092,480, U[1,1000], seeded sources",
    "rmat": "config 3: RMAT scale 24 edge factor 16 (Graph500 abcd), n=16,777,216 m=268,435,456, U[1,255], "
            "seeded sources",
    "er": "config 4: Erdos-Renyi directed G(2^24, 32*2^24), m=536,870,912, U[1,2^20], seeded sources",
}
METRIC = "GTEPS (E_dij per second) and ms/source; config 5 multi-source batch on 1/2/4/8 GPUs"
L2_BYTES = 126 * 2**20
GATHER_PEAK_G = 280.0  # measured random L2 gather rate (tools/gather_bench.cu, this pool's B200)
BATCH_K = 512
E2E_CHUNK = 64  # sources per host-output sssp_run_batch call of the e2e pass (64 x 134 MB = 8.6 GB pinned):
                # each call ends with its last copies unoverlapped (16: e2e 65.6-67.7, 64: 72.5-74.8 GTEPS)


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def ncu_traffic(config, block, grid):
    """DRAM bytes per launch of the persistent kernel from the committed ncu --set full
    summary -- only if that capture is of the same launch shape as the benched runs."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_summary.json")) as f:
            d = json.load(f)
    except Exception:
        return None, "no profiles/ncu_summary.json"
    e = d.get(config)
    if not e:
        return None, f"no ncu capture for {config}"
    shape = (e.get("block"), e.get("grid"))
    if shape != (block, grid):
        return None, f"ncu capture shape {shape} != benched (block, grid) {(block, grid)}: refused"
    return e.get("dram_bytes_per_launch"), f"profiles/ncu_summary.json [{config}] ({e.get('round', '?')})"


def host_info():
    model = platform.processor() or ""
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count()}


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None
        return self

    def __exit__(self, *a):
        self.rows = []
        if self.p is None:
            return
        time.sleep(0.25)
        self.p.terminate()
        try:
            out, _ = self.p.communicate(timeout=5)
        except Exception:
            self.p.kill()
            out = ""
        for line in out.splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) >= 9:
                self.rows.append(f)

    def summary(self):
        rows = getattr(self, "rows", [])
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        # under load only (the sampler also sees the idle tail of the region)
        busy = sorted(sm)[len(sm) // 4:] if len(sm) >= 8 else sm
        return {"sm_mhz": statistics.median(busy) if busy else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def batch_sources(g):
    return gg.sources(g, BATCH_K, gg.CONFIGS["batch"]["source_seed"])


# ------------------------------------------------------------------ the oracle, on host cores
def oracle_pool(g, srcs, threads):
    """Run the oracle on ``srcs`` with ``threads`` host threads (ctypes releases the GIL,
    so each thread runs one Dijkstra on its own core); returns (seconds, E_dij sum)."""
    import oracle
    todo = list(int(s) for s in srcs)
    lock = threading.Lock()
    E = [0]

    def work():
        while True:
            with lock:
                if not todo:
                    return
                s = todo.pop()
            _, _, e = oracle.dijkstra(g, s)
            with lock:
                E[0] += e

    ts = [threading.Thread(target=work) for _ in range(threads)]
    t0 = time.perf_counter()
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    return time.perf_counter() - t0, E[0]


def cpu_baseline_single(g, src, name):
    import oracle
    t0 = time.perf_counter()
    _, _, e = oracle.dijkstra(g, int(src))
    dt = time.perf_counter() - t0
    return {"value": e / dt / 1e9, "unit": "GTEPS", "cores": 1, "kind": "oracle",
            "sample": f"1 full single-source run on the {name} graph (binary-heap Dijkstra, C, 1 thread, "
                      f"{dt:.2f} s)", **host_info()}


def cpu_baseline_batch(g, srcs):
    P = min(len(srcs), os.cpu_count() or 1)
    dt, E = oracle_pool(g, srcs[:P], P)
    return {"value": E / dt / 1e9, "unit": "GTEPS", "cores": P, "kind": "oracle",
            "sample": f"{P} of the batch's sources, one per host thread on {P} threads at once "
                      f"(binary-heap Dijkstra, C), {dt:.2f} s wall", **host_info()}


# ------------------------------------------------------------------ reference arm
def run_reference(args, world, rank):
    if rank != 0:
        return 0
    cfg = args.config
    g = gg.make("rmat" if cfg == "batch" else cfg)
    P = os.cpu_count() or 1
    if cfg == "batch":
        srcs = batch_sources(g)
        per = min(P, len(srcs))
    else:
        srcs = gg.config_sources(cfg, g, args.warmup + args.steps + 1)
        per = 1
    import oracle
    # warm-up: one source whatever W is (it only pages the graph in; a CPU program has no
    # device state to warm, and each RMAT-24 source costs seconds)
    if args.warmup:
        oracle.dijkstra(g, int(srcs[0]))
    total_s, E = 0.0, 0
    for k in range(args.steps):
        sample = [srcs[(k * per + j) % len(srcs)] for j in range(per)]
        dt, e = oracle_pool(g, sample, per)
        total_s += dt
        E += e
    v = E / total_s / 1e9
    units = args.steps * per
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "GTEPS", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": total_s * 1e3 / args.steps,
        "higher_is_better": True, "scaling": "strong" if cfg == "batch" else "weak", "vs_baseline": None,
        "dtype": "u64", "data": "synthetic",
        "config": {"workload": WORKLOADS[cfg], "name": cfg, "n": g.n, "m": g.m},
        "ms_per_source": total_s * 1e3 / units * per,
        "cpu_baseline": {"value": v, "unit": "GTEPS", "cores": per, "kind": "oracle",
                         "sample": f"each step: {per} source(s) of the {cfg} workload on {per} host thread(s) "
                                   "at once (binary-heap Dijkstra, C)", **host_info()},
        "e2e": {"value": v, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def alg_bytes(st):
    """SURVEY §8(d) algorithmic bytes of the persistent kernel with this layout: 12 B per arc
    relaxed (8 B {col,w} + 4 B dist gather) + 20 B per vertex expanded."""
    return 12 * st["edges_relaxed"] + 20 * st["vertices_processed"]


def roofline(bytes_, ms, traffic, note, launches):
    hbm, peak_kind = peaks()
    achieved = bytes_ / (ms / 1e3) / 1e9 if ms > 0 else 0.0
    return {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s", "frac": achieved / hbm,
            "traffic": traffic, "traffic_source": note, "peak_kind": peak_kind, "kernel": "adds_persistent_kernel",
            "alg_bytes_per_launch": bytes_ / max(1, launches), "launches": launches}


def run_singles(args, sssp, torch, dev, local):
    """Configs 2-4 (single-source, one GPU): per config W warm-up + K timed sources."""
    res = {}
    for cfg in args.singles:
        g = gg.make(cfg)
        srcs = gg.config_sources(cfg, g, args.single_warmup + args.single_steps)
        G = sssp.Graph.from_csr(g, device=local)
        out = torch.empty(g.n, dtype=torch.int64, device=dev)
        stream = torch.cuda.current_stream(dev)
        for i in range(args.single_warmup):
            G.run(int(srcs[i]), out=out, stream=stream)
        acc = {k: 0 for k in ("edges_relaxed", "vertices_processed", "reach_edges", "reachable", "pushes")}
        kms, launches, lst = 0.0, 0, None
        torch.cuda.synchronize(dev)
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        ev[0].record(stream)
        for i in range(args.single_steps):
            G.run(int(srcs[args.single_warmup + i]), out=out, stream=stream)
            lst = G.stats()
            for k in acc:
                acc[k] += lst[k]
            kms += lst["kernel_ms"]
            launches += 1 + lst["retries"]
        ev[1].record(stream)
        torch.cuda.synchronize(dev)
        T = ev[0].elapsed_time(ev[1])
        traffic, note = ncu_traffic(cfg, lst["block_threads"], lst["grid_ctas"])
        k = args.single_steps
        rand_acc = (acc["edges_relaxed"] + acc["pushes"] + 3 * acc["vertices_processed"]) / k
        res[cfg] = {
            "workload": WORKLOADS[cfg], "n": g.n, "m": g.m, "sources": k,
            "ms_per_source": T / k, "kernel_ms_per_source": kms / k,
            "value": acc["reach_edges"] / (T / 1e3) / 1e9, "unit": "GTEPS",
            "work_efficiency": {"edges": acc["edges_relaxed"] / max(1, acc["reach_edges"]),
                                "vertices": acc["vertices_processed"] / max(1, acc["reachable"])},
            "delta_log2": {"init": lst["init_delta_log2"], "final": lst["final_delta_log2"]},
            "grid_ctas": lst["grid_ctas"], "block_threads": lst["block_threads"],
            "roofline": roofline(alg_bytes(acc), kms, traffic, note, launches),
            "gather_roofline": {"bound": "l2_random_access", "achieved": rand_acc / (kms / k / 1e3) / 1e9,
                                "unit": "G accesses/s", "peak": GATHER_PEAK_G,
                                "frac": rand_acc / (kms / k / 1e3) / 1e9 / GATHER_PEAK_G},
            "gpu_launches": 3 * launches,
        }
        if not args.no_cpu_baseline:
            res[cfg]["cpu_baseline"] = cpu_baseline_single(g, srcs[-1], cfg)
        del out
        G.close()
        del g
        torch.cuda.empty_cache()
    return res


def run_ours(args, world, rank, local):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_wangfl21_b200 as sssp
    from paper_conf_ppopp_wangfl21_b200.distributed import barrier, partition, run_batch_distributed

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    cfg = args.config
    stream = torch.cuda.current_stream(dev)
    g = gg.make("rmat" if cfg == "batch" else cfg)
    if cfg == "batch":
        allsrc = batch_sources(g)
    else:  # a single-source config as the main line: K sources per rank (weak scaling, replicas)
        allsrc = gg.config_sources(cfg, g, (args.warmup + args.steps) * world)
    mine = partition(allsrc, world, rank)
    opts = dict(device=local, concurrent_sources=args.concurrency)
    if args.algorithm == "nearfar":
        opts["algorithm"] = sssp.SSSP_ALGO_NEAR_FAR
    G = sssp.Graph.from_csr(g, **opts)
    if cfg == "batch":
        step_srcs = [allsrc] * (args.warmup + args.steps)
    else:  # one source per rank per step
        step_srcs = [allsrc[i * world:(i + 1) * world] for i in range(args.warmup + args.steps)]
    per_rank = max(len(partition(s, world, rank)) for s in step_srcs)
    D = torch.empty((per_rank, g.n), dtype=torch.int64, device=dev)

    def step(srcs):
        return run_batch_distributed(G, srcs, out=D, stream=stream, device=dev)

    for i in range(args.warmup):
        step(step_srcs[i])

    # timed region: K steps, barrier + synchronize on both sides, CUDA events on the run stream
    tot = {k: 0.0 for k in ("edges_relaxed", "vertices_processed", "reach_edges", "reachable", "pushes", "runs",
                            "retries")}
    my = {k: 0.0 for k in tot}
    kms, launches = 0.0, 0
    with ClockSampler(local) as clk:
        barrier(None, dev)
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        ev[0].record(stream)
        for i in range(args.steps):
            r = step(step_srcs[args.warmup + i])
            for k in tot:
                tot[k] += r["stats"][k]
            st = G.stats()
            for k in my:
                my[k] += st.get(k, 0)
            kms += st["kernel_ms"]
            launches += int(st["runs"] + st["retries"])
        ev[1].record(stream)
        barrier(None, dev)
    t_ms = ev[0].elapsed_time(ev[1])
    tmax = torch.tensor([t_ms], dtype=torch.float64, device=dev)
    lt = torch.tensor([float(launches)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        dist.all_reduce(lt, op=dist.ReduceOp.SUM)
    T = float(tmax.item())
    last = G.stats()
    units = int(tot["runs"])
    value = tot["reach_edges"] / (T / 1e3) / 1e9

    # the single-source configs run next, on a quiet host (after the e2e pass's 68 GB of copies
    # and the CPU baseline's threads their device-timed runs picked up host-side gaps)
    singles = None
    if rank == 0 and world == 1 and args.singles:
        singles = run_singles(args, sssp, torch, dev, local)

    # e2e through the public C ABI with host buffers: the sources go in and every full distance
    # vector comes back to pinned host memory inside the call (sssp_run_batch on chunks of
    # E2E_CHUNK sources into one pinned host buffer; the library overlaps each row's copy with
    # the next sources' compute)
    e2e = None
    if args.e2e_steps > 0:
        e2e_src = mine if cfg == "batch" else mine[: args.e2e_steps]
        chunk = max(1, min(args.e2e_chunk, len(e2e_src)))
        dist_h = torch.empty((chunk, g.n), dtype=torch.int64).pin_memory()
        barrier(None, dev)
        t0 = time.perf_counter()
        Ee = 0
        for c0 in range(0, len(e2e_src), chunk):
            part = np.ascontiguousarray(e2e_src[c0:c0 + chunk], dtype=np.uint32)
            sssp._check(sssp.lib().sssp_run_batch(G._h, part.ctypes.data, len(part), dist_h.data_ptr(),
                                                  sssp._stream_ptr(stream)))
            Ee += G.stats()["reach_edges"]
        torch.cuda.synchronize(dev)
        te = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        ee = torch.tensor([float(Ee)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
            dist.all_reduce(ee, op=dist.ReduceOp.SUM)
        e2e = {"value": ee.item() / te.item() / 1e9, "unit": "GTEPS", "h2d_bytes_per_step": 4 * len(e2e_src),
               "d2h_bytes_per_step": int(8 * g.n * len(e2e_src)), "steps": 1,
               "path": f"graph resident; sssp_run_batch(chunks of {chunk} sources, pinned host dist_out) over the "
                       "rank's slice: one pass, every distance vector copied to the host inside the call "
                       "(per-slot device staging rows, copies overlapped with the next sources)"}
        del dist_h
        if hasattr(torch._C, "_host_emptyCache"):
            torch._C._host_emptyCache()  # (return the pinned staging memory)
    del D
    torch.cuda.empty_cache()

    line = None
    if rank == 0:
        traffic, note = ncu_traffic(cfg, last["block_threads"], last["grid_ctas"])
        # rank 0's launches over rank 0's device time of the K steps (with c sources in
        # flight the launches overlap, so the batch time -- not the per-launch time -- is
        # what one GPU sustained)
        rf = roofline(alg_bytes(my), t_ms, traffic, note, launches)
        rf["note"] = (f"{args.concurrency} sources in flight per GPU on 1/{args.concurrency} of the SMs each: "
                      "achieved = rank 0's algorithmic bytes / rank 0's device time of the K steps")
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            cpu = cpu_baseline_batch(g, mine) if cfg == "batch" else cpu_baseline_single(g, mine[-1], cfg)
        csr_bytes = g.nbytes()
        line = {
            "metric": METRIC, "value": value, "unit": "GTEPS", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": T / args.steps, "higher_is_better": True,
            "scaling": "strong" if cfg == "batch" else "weak", "vs_baseline": None,
            "dtype": f"u{last['dist_bits']}", "data": "synthetic (seeded generator, graphgen/)",
            "config": {"workload": WORKLOADS[cfg], "name": cfg, "n": g.n, "m": g.m,
                       "sources_per_step": int(units / args.steps),
                       "parallelism": f"source-partitioned x{world}, CSR replicated",
                       "l2": f"inputs larger than L2 (CSR {csr_bytes / 2**20:.0f} MiB > 126 MiB), no flush"
                       if csr_bytes > L2_BYTES else "small input (L2-resident)",
                       "grid_ctas": last["grid_ctas"], "block_threads": last["block_threads"],
                       "algorithm": args.algorithm, "concurrent_sources": args.concurrency},
            "ms_per_source": T / max(1, units / world) if cfg != "batch" else T / max(1, units),
            "work_efficiency": {"edges": tot["edges_relaxed"] / max(1, tot["reach_edges"]),
                                "vertices": tot["vertices_processed"] / max(1, tot["reachable"])},
            "delta_log2": {"init": last["init_delta_log2"], "final": last["final_delta_log2"]},
            "roofline": rf,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(3 * lt.item()),
            "retries": int(tot["retries"]),
            "clocks": clk.summary(),
        }
    del G, g
    torch.cuda.empty_cache()
    if singles is not None:
        line["singles"] = singles
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="batch", choices=list(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3, help="0 = skip the host-buffer e2e pass")
    ap.add_argument("--e2e-chunk", type=int, default=E2E_CHUNK, help="sources per host-output batch call (e2e)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-singles", action="store_true", help="skip the single-source configs 2-4 (N=1 only)")
    ap.add_argument("--single-steps", type=int, default=5)
    ap.add_argument("--single-warmup", type=int, default=3)
    ap.add_argument("--algorithm", default="adds", choices=["adds", "nearfar"],
                    help="nearfar = the paper's BSP comparison system (ablation, NEXT-2)")
    ap.add_argument("--concurrency", type=int, default=4,
                    help="sources in flight per GPU (NEXT-1, options.concurrent_sources)")
    args = ap.parse_args()
    args.singles = [] if args.no_singles or args.config != "batch" else ["road", "rmat", "er"]
    world, rank, local = dist_env()
    if args.impl == "reference":
        return run_reference(args, world, rank)
    return run_ours(args, world, rank, local)


if __name__ == "__main__":
    sys.exit(main())

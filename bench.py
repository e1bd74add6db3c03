#!/usr/bin/env python
"""Benchmark of the ADDS SSSP hot path on B200 (one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config road|rmat|er|grid64|batch]
                    [--impl ours|reference]

A step = one single-source SSSP (init + persistent ADDS kernel + finalize)
through the C ABI on a graph resident in HBM, inputs already on the device.
Default workload = BASELINE.json configs[1] (4096x4096 perturbed grid,
U[1,1000]).  Under torchrun each rank runs its own sources on its own GPU with
its own replica of the graph (weak scaling, no data-path collective); the
timed region is bracketed by barrier + synchronize and the max over ranks is
taken.  ``value`` = GTEPS = sum over ranks/steps of E_dij (arcs out of
reachable vertices, Graph500-style algorithmic TEPS, reading R2) / time.

--impl reference times the CPU oracle (binary-heap Dijkstra, the paper's own
serial baseline P:268) on the same workload; it is one of the three places
allowed to run oracle/.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402

WORKLOADS = {
    "grid64": "64x64 grid, 4-neighbour, U[1,100], source 0",
    "road": "4096x4096 perturbed grid (road-like), n=16,777,216 m=67,092,480, U[1,1000], seeded sources",
    "rmat": "RMAT scale 24 edge factor 16 (Graph500 abcd), n=16,777,216 m=268,435,456, U[1,255], seeded sources",
    "er": "Erdos-Renyi directed G(2^24, 32*2^24), m=536,870,912, U[1,2^20], seeded sources",
    "batch": "RMAT scale 24 edge factor 16, 512 seeded sources partitioned across ranks",
}
METRIC = "GTEPS (E_dij per second) and ms/source, single-source SSSP"
L2_BYTES = 126 * 2**20
GATHER_PEAK_G = 280.0  # measured random L2 gather rate (tools/gather_bench.cu, this pool's B200)


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def ncu_traffic(config):
    """dram bytes per launch of the persistent kernel from the committed ncu --set full summary."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_summary.json")) as f:
            d = json.load(f)
        # a batch launch is one RMAT-24 source (on 1/c of the SMs): the rmat capture's bytes
        return d.get("rmat" if config == "batch" else config, {}).get("dram_bytes_per_launch")
    except Exception:
        return None


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
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def dist_init():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def build_graph(config):
    name = "rmat" if config == "batch" else config
    return gg.make(name)


def step_sources(config, g, world, rank, count):
    if config == "grid64":
        return np.zeros(count, dtype=np.uint32)
    seed = gg.CONFIGS[config]["source_seed"]
    allsrc = gg.sources(g, count * world, seed)
    return allsrc[rank::world][:count]


# ------------------------------------------------------------------ reference arm
def run_reference(args, world, rank):
    if rank != 0:
        return 0
    import oracle
    g = build_graph(args.config)
    srcs = step_sources(args.config, g, 1, 0, args.warmup + args.steps)
    for i in range(args.warmup):
        oracle.dijkstra(g, int(srcs[i]))
    t0 = time.perf_counter()
    E = 0
    for i in range(args.steps):
        _, _, e = oracle.dijkstra(g, int(srcs[args.warmup + i]))
        E += e
    dt = time.perf_counter() - t0
    v = E / dt / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "GTEPS", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": WORKLOADS[args.config], "name": args.config, "n": g.n, "m": g.m},
        "cpu_baseline": {"value": v, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                         "sample": f"{args.steps} full single-source runs of the {args.config} graph "
                                   "(binary-heap Dijkstra, C, 1 thread)"},
        "e2e": {"value": v, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def run_ours(args, world, rank, local):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_wangfl21_b200 as sssp

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)

    g = build_graph(args.config)
    n_src = args.warmup + args.steps
    if args.config == "batch":
        per_rank = 512 // world
        srcs = gg.sources(g, 512, gg.CONFIGS["batch"]["source_seed"])[rank::world]
        n_src = len(srcs)
    else:
        srcs = step_sources(args.config, g, world, rank, n_src)
    opts = dict(device=local, algorithm=sssp.SSSP_ALGO_NEAR_FAR if args.algorithm == "nearfar" else sssp.SSSP_ALGO_ADDS)
    if args.config == "batch":
        opts["concurrent_sources"] = args.concurrency
    G = sssp.Graph.from_csr(g, **opts)
    stream = torch.cuda.current_stream(dev)
    out = torch.empty(g.n, dtype=torch.int64, device=dev)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    # warm-up
    for i in range(args.warmup):
        G.run(int(srcs[i % len(srcs)]), out=out, stream=stream)

    # timed region
    kms, E_dij, V_dij, E_gpu, V_gpu, pushes, retries = 0.0, 0, 0, 0, 0, 0, 0
    launches = 0
    with ClockSampler(local) as clk:
        barrier()
        ev0 = torch.cuda.Event(enable_timing=True)
        ev1 = torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        if args.config == "batch":
            D = torch.empty((len(srcs), g.n), dtype=torch.int64, device=dev)
            reps = args.steps
            for _ in range(reps):
                G.run_batch(srcs, out=D, stream=stream)
                st = G.stats()
                kms += st["kernel_ms"]
                E_dij += st["reach_edges"]
                V_dij += st["reachable"]
                E_gpu += st["edges_relaxed"]
                V_gpu += st["vertices_processed"]
                pushes += st["pushes"]
                retries += st["retries"]
                launches += 3 * (st["runs"] + st["retries"])
            units = reps * len(srcs)
        else:
            for i in range(args.steps):
                G.run(int(srcs[args.warmup + i]), out=out, stream=stream)
                st = G.stats()
                kms += st["kernel_ms"]
                E_dij += st["reach_edges"]
                V_dij += st["reachable"]
                E_gpu += st["edges_relaxed"]
                V_gpu += st["vertices_processed"]
                pushes += st["pushes"]
                retries += st["retries"]
                launches += 3 * (1 + st["retries"])
            units = args.steps
        ev1.record(stream)
        barrier()
    t_ms = ev0.elapsed_time(ev1)
    last = G.stats()

    tot = torch.tensor([E_dij, E_gpu, V_dij, V_gpu, launches], dtype=torch.float64, device=dev)
    tmax = torch.tensor([t_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.SUM)
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
    E_all, Eg_all, V_all, Vg_all, _ = tot.tolist()
    T = tmax.item()
    value = E_all / (T / 1e3) / 1e9

    # e2e: same metric through the public C ABI from pinned HOST buffers every step:
    # graph upload (create) + run into pinned host dist + destroy
    e2e = None
    if args.e2e_steps > 0 and args.config == "batch":
        # batch served to the host: the rank's sources (host array) go in, every
        # source's full distance vector comes back to pinned host memory inside the
        # call (68.7 GB for the whole batch does not fit in pinned memory at once, so
        # each row is streamed out as it completes); one pass over the rank's slice
        dist_h = torch.empty(g.n, dtype=torch.int64).pin_memory()
        barrier()
        t0 = time.perf_counter()
        Ee = 0
        for s in srcs:
            sssp._check(sssp.lib().sssp_run(G._h, int(s), dist_h.data_ptr(), sssp._stream_ptr(stream)))
            Ee += G.stats()["reach_edges"]
        torch.cuda.synchronize(dev)
        te = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        ee = torch.tensor([float(Ee)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
            dist.all_reduce(ee, op=dist.ReduceOp.SUM)
        e2e = {"value": ee.item() / te.item() / 1e9, "unit": "GTEPS", "h2d_bytes_per_step": 4 * len(srcs),
               "d2h_bytes_per_step": int(8 * g.n * len(srcs)), "steps": 1,
               "path": "resident graph; per source sssp_run(source, host dist_out) over the rank's slice"}
    if args.e2e_steps > 0 and args.config != "batch":
        off_h = torch.from_numpy(g.row_offsets.view(np.int64)).pin_memory()
        col_h = torch.from_numpy(g.col.view(np.int32)).pin_memory()
        w_h = torch.from_numpy(g.w.view(np.int32)).pin_memory()
        dist_h = torch.empty(g.n, dtype=torch.int64).pin_memory()
        k_e = min(args.e2e_steps, args.steps)
        barrier()
        t0 = time.perf_counter()
        Ee = 0
        for i in range(k_e):
            H = sssp.Graph(off_h, col_h, w_h, device=local)
            sssp._check(sssp.lib().sssp_run(H._h, int(srcs[args.warmup + i]), dist_h.data_ptr(),
                                            sssp._stream_ptr(stream)))
            Ee += H.stats()["reach_edges"]
            H.close()
        torch.cuda.synchronize(dev)
        te = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        ee = torch.tensor([float(Ee)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
            dist.all_reduce(ee, op=dist.ReduceOp.SUM)
        e2e = {"value": ee.item() / te.item() / 1e9, "unit": "GTEPS",
               "h2d_bytes_per_step": int(g.row_offsets.nbytes + g.col.nbytes + g.w.nbytes),
               "d2h_bytes_per_step": int(8 * g.n), "steps": k_e,
               "path": "sssp_graph_create(pinned host CSR) + sssp_run(host dist_out) + destroy"}
        # serving shape: the graph stays resident (uploaded once, like model weights), every
        # query is a source in and a full distance vector out to pinned host memory
        barrier()
        t0 = time.perf_counter()
        Er = 0
        for i in range(args.steps):
            sssp._check(sssp.lib().sssp_run(G._h, int(srcs[args.warmup + i]), dist_h.data_ptr(),
                                            sssp._stream_ptr(stream)))
            Er += G.stats()["reach_edges"]
        torch.cuda.synchronize(dev)
        tr = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        er = torch.tensor([float(Er)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(tr, op=dist.ReduceOp.MAX)
            dist.all_reduce(er, op=dist.ReduceOp.SUM)
        e2e["resident_graph"] = {"value": er.item() / tr.item() / 1e9, "unit": "GTEPS", "steps": args.steps,
                                 "h2d_bytes_per_step": 0, "d2h_bytes_per_step": int(8 * g.n),
                                 "path": "sssp_run(resident graph, host dist_out): source in, distances "
                                         "copied to pinned host memory inside the call"}

    if rank == 0:
        hbm, peak_kind = peaks()
        per_launch_ms = kms / max(1, (units if args.config != "batch" else units))
        # algorithmic bytes of the persistent kernel:
        # 12 B per arc relaxed (8 B {col,w} + 4 B dist gather) + 20 B per vertex expanded
        alg_bytes = (12 * E_gpu + 20 * V_gpu) / max(1, units)
        achieved = alg_bytes / (per_launch_ms / 1e3) / 1e9
        # the bound actually binding: random 4-byte L2 accesses, one
        # distinct line each -- a dist gather per arc, an atomic per push, and
        # dist + row-offset + item accesses per popped item
        rand_acc = (E_gpu + pushes + 3 * V_gpu) / max(1, units)
        rand_rate = rand_acc / (per_launch_ms / 1e3) / 1e9
        traffic = ncu_traffic(args.config)
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            import oracle
            t0 = time.perf_counter()
            _, _, e = oracle.dijkstra(g, int(srcs[args.warmup % len(srcs)]))
            dt = time.perf_counter() - t0
            cpu = {"value": e / dt / 1e9, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                   "sample": f"1 full single-source run on the {args.config} graph "
                             f"(binary-heap Dijkstra, C, 1 thread, {dt:.2f} s)"}
        csr_bytes = g.row_offsets.nbytes + g.col.nbytes + g.w.nbytes
        line = {
            "metric": METRIC, "value": value, "unit": "GTEPS", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": T / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": f"u{last['dist_bits']}", "data": "synthetic",
            "config": {"workload": WORKLOADS[args.config], "name": args.config, "n": g.n, "m": g.m,
                       "sources_per_step_per_rank": (len(srcs) if args.config == "batch" else 1),
                       "parallelism": f"source-partitioned x{world} (graph replicated)",
                       "l2": f"inputs larger than L2 (CSR {csr_bytes / 2**20:.0f} MiB > 126 MiB), no flush"
                       if csr_bytes > L2_BYTES else "small input (L2-resident)",
                       "grid_ctas": last["grid_ctas"], "block_threads": last["block_threads"],
                       "algorithm": args.algorithm,
                       "concurrent_sources": (args.concurrency if args.config == "batch" else 1)},
            "ms_per_source": T / units,
            "work_efficiency": {"edges": Eg_all / max(1, E_all), "vertices": Vg_all / max(1, V_all)},
            "delta_log2": {"init": last["init_delta_log2"], "final": last["final_delta_log2"]},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                         "frac": achieved / hbm, "traffic": traffic, "peak_kind": peak_kind,
                         "kernel": "adds_persistent_kernel", "kernel_ms_avg": per_launch_ms,
                         "alg_bytes_per_launch": alg_bytes},
            "gather_roofline": {"bound": "l2_random_access", "achieved": rand_rate, "unit": "G accesses/s",
                                "peak": GATHER_PEAK_G, "frac": rand_rate / GATHER_PEAK_G,
                                "peak_source": "tools/gather_bench.cu on B200: random 4-byte gathers, "
                                               "67 MB L2-resident array, 1184x256 threads"},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(launches),
            "retries": int(retries),
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=8)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="road", choices=list(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--algorithm", default="adds", choices=["adds", "nearfar"],
                    help="nearfar = the paper's BSP comparison system (ablation, NEXT-2)")
    ap.add_argument("--concurrency", type=int, default=2,
                    help="sources in flight per GPU for --config batch (measured 1/2/4/8: 44.9/46.6/44.3/25.7 GTEPS)")
    args = ap.parse_args()
    world, rank, local = dist_init()
    if args.impl == "reference":
        return run_reference(args, world, rank)
    return run_ours(args, world, rank, local)


if __name__ == "__main__":
    sys.exit(main())

"""Multi-GPU multi-source batches (BASELINE config 5).

A single SSSP does not shard (the paper is single-GPU; Delta-stepping's bucket
order is a global dependency), so only batches of independent sources are
partitioned: sources are dealt round-robin to ranks (``sources[rank::world]``),
each rank holds a full replica of the CSR and runs its slice with
``sssp_run_batch``.  There is no collective on the data path.  After the
compute, one all-reduce sums the work counters and one takes the max of the
per-rank device times; an optional gather of the distance rows to one rank is a
separate, separately timed collective.

``run_batch_distributed`` is the one rank loop: ``bench.py`` drives it with the
device runner (``Graph.run_batch``) over NCCL, and tests/test_distributed.py
drives the same function with a CPU runner over gloo at world sizes 2 and 4.
"""
from __future__ import annotations

import time

import numpy as np

COUNTERS = ["edges_relaxed", "vertices_processed", "reach_edges", "reachable", "pushes", "runs", "retries"]


def partition(sources, world: int, rank: int) -> np.ndarray:
    """Round-robin slice of the source list owned by ``rank``."""
    src = np.asarray(sources, dtype=np.uint32)
    return src[rank::world].copy()


def owner_and_row(i: int, world: int):
    """Where global source index i lives: (rank, row within that rank's block)."""
    return i % world, i // world


class _Clock:
    """Device time on ``stream`` (CUDA events) for a cuda device, wall time otherwise."""

    def __init__(self, device, stream):
        import torch
        self.cuda = device is not None and torch.device(device).type == "cuda"
        if self.cuda:
            self.stream = stream if stream is not None else torch.cuda.current_stream(device)
            self.ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]

    def start(self):
        if self.cuda:
            self.ev[0].record(self.stream)
        else:
            self.t0 = time.perf_counter()

    def stop(self):
        if self.cuda:
            self.ev[1].record(self.stream)
        else:
            self.t1 = time.perf_counter()

    def ms(self) -> float:
        if self.cuda:
            self.ev[1].synchronize()
            return float(self.ev[0].elapsed_time(self.ev[1]))
        return (self.t1 - self.t0) * 1e3


def barrier(group=None, device=None):
    """dist.barrier (when initialised) + a device synchronize (cuda devices)."""
    import torch
    import torch.distributed as dist
    if dist.is_initialized():
        dist.barrier(group=group)
    if device is not None and torch.device(device).type == "cuda":
        torch.cuda.synchronize(device)


def run_batch_distributed(graph, sources, group=None, gather_to=None, runner=None, device=None, out=None,
                          stream=None):
    """Run every source of ``sources`` once across the ranks of ``group``.

    graph     : a ``paper_conf_ppopp_wangfl21_b200.Graph`` on this rank's GPU (unused with ``runner``)
    runner    : callable(slice) -> (dist [k, n] tensor, stats dict); default
                ``graph.run_batch(slice, out=out, stream=stream)`` + ``graph.stats()``
    device    : where the counters live and how time is taken (cuda: CUDA events on
                ``stream``; cpu: wall clock); default the graph's GPU
    gather_to : rank that receives every row (``full``, [len(sources), n] in source
                order), timed separately as ``gather_ms``; None = no gather

    The compute is bracketed by barrier + synchronize on both sides.  Returns dict(
    local=this rank's rows, sources=its slice, stats=counters summed over ranks,
    max_ms=max over ranks of the device time of the compute, local_ms=this rank's,
    full / gather_ms when gathered).
    """
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    mine = partition(sources, world, rank)
    if device is None:
        device = torch.device("cuda", graph.device)
    if runner is None:
        def runner(sl):
            if len(sl) == 0:
                return torch.empty((0, graph.n), dtype=torch.int64, device=device), {}
            o = None if out is None else out[: len(sl)]
            d = graph.run_batch(sl, out=o, stream=stream)
            return d, graph.stats()
    clock = _Clock(device, stream)
    barrier(group, device)
    clock.start()
    local, st = runner(mine)
    clock.stop()
    barrier(group, device)
    local_ms = clock.ms()
    counts = torch.tensor([float(st.get(k, 0)) for k in COUNTERS], dtype=torch.float64, device=device)
    tmax = torch.tensor([local_ms], dtype=torch.float64, device=device)
    if world > 1:
        dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX, group=group)
    res = {"local": local, "sources": mine, "stats": dict(zip(COUNTERS, counts.tolist())),
           "max_ms": float(tmax.item()), "local_ms": local_ms}
    if gather_to is not None:
        t0 = time.perf_counter()
        res["full"] = gather_rows(local, len(sources), world, rank, gather_to, group)
        res["gather_ms"] = (time.perf_counter() - t0) * 1e3
    return res


def gather_rows(local, k: int, world: int, rank: int, dst: int, group=None):
    """Collect every rank's rows on rank ``dst`` in global source order (other ranks get None)."""
    import torch
    import torch.distributed as dist

    per = (k + world - 1) // world
    n = local.shape[1]
    pad = torch.full((per, n), -1, dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    if world > 1:
        bufs = [torch.empty_like(pad) for _ in range(world)] if rank == dst else None
        dist.gather(pad, gather_list=bufs, dst=dst, group=group)
    else:
        bufs = [pad]
    if rank != dst:
        return None
    full = torch.empty((k, n), dtype=local.dtype, device=local.device)
    for i in range(k):
        r, row = owner_and_row(i, world)
        full[i] = bufs[r][row]
    return full

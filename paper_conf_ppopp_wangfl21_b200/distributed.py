"""Multi-GPU multi-source batches (BASELINE config 5).

A single SSSP does not shard (the paper is single-GPU; Delta-stepping's bucket
order is a global dependency), so only batches of independent sources are
partitioned: sources are dealt round-robin to ranks (``sources[rank::world]``),
each rank holds a full replica of the CSR and runs its slice with
``sssp_run_batch``.  There is no collective on the data path; NCCL is used
only after the compute for an all-reduce of the work counters and the max
device time, and (optionally, timed separately) to gather distance rows.

The partition / reassembly logic is independent of the device runner so it can
be tested with ``gloo`` on CPU (tests/test_distributed.py).
"""
from __future__ import annotations

import numpy as np


def partition(sources, world: int, rank: int) -> np.ndarray:
    """Round-robin slice of the source list owned by ``rank``."""
    src = np.asarray(sources, dtype=np.uint32)
    return src[rank::world].copy()


def owner_and_row(i: int, world: int):
    """Where global source index i lives: (rank, row within that rank's block)."""
    return i % world, i // world


def run_batch_distributed(graph, sources, group=None, gather: bool = False, runner=None, device=None):
    """Run every source of ``sources`` once across the ranks of ``group``.

    graph   : a ``paper_conf_ppopp_wangfl21_b200.Graph`` on this rank's GPU
              (ignored when ``runner`` is given)
    runner  : optional callable(slice) -> (dist [k, n] tensor, stats dict);
              defaults to ``graph.run_batch`` + ``graph.stats``
    gather  : also assemble the full [len(sources), n] result on every rank
              (all_gather; a collective AFTER the compute, reported separately)

    Returns dict(local=dist of this rank's slice, sources=slice, stats=summed
    counters over ranks, max_ms=max device time over ranks, full=... if gather).
    """
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    mine = partition(sources, world, rank)
    if runner is None:
        def runner(sl):
            if len(sl) == 0:
                return torch.empty((0, graph.n), dtype=torch.int64, device=f"cuda:{graph.device}"), {}
            d = graph.run_batch(sl)
            return d, graph.stats()
    local, st = runner(mine)
    dev = local.device if device is None else device
    keys = ["edges_relaxed", "vertices_processed", "reach_edges", "reachable", "pushes", "runs"]
    counts = torch.tensor([float(st.get(k, 0)) for k in keys], dtype=torch.float64, device=dev)
    tmax = torch.tensor([float(st.get("total_ms", 0.0))], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX, group=group)
    out = {"local": local, "sources": mine, "stats": dict(zip(keys, counts.tolist())), "max_ms": tmax.item()}
    if gather:
        k = len(sources)
        per = (k + world - 1) // world
        n = local.shape[1]
        pad = torch.full((per, n), -1, dtype=local.dtype, device=local.device)
        pad[: local.shape[0]] = local
        if world > 1:
            bufs = [torch.empty_like(pad) for _ in range(world)]
            dist.all_gather(bufs, pad, group=group)
        else:
            bufs = [pad]
        full = torch.empty((k, n), dtype=local.dtype, device=local.device)
        for i in range(k):
            r, row = owner_and_row(i, world)
            full[i] = bufs[r][row]
        out["full"] = full
    return out

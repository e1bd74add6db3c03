"""Multi-rank (world_size 2, gloo, CPU) tests of the source-partitioned batch
path: partition covers every source exactly once, counters
sum over ranks, and the optional gather reassembles rows in source order.
The per-rank runner here is the CPU oracle (tests may use it); the device
runner is exercised by the GPU tests and bench.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen as gg
import oracle
from paper_conf_ppopp_wangfl21_b200.distributed import owner_and_row, partition, run_batch_distributed


def test_partition_covers_each_source_once():
    src = np.arange(37, dtype=np.uint32) * 3
    for world in (1, 2, 3, 8):
        parts = [partition(src, world, r) for r in range(world)]
        allp = np.concatenate(parts)
        assert sorted(allp.tolist()) == sorted(src.tolist())
        for i in range(len(src)):
            r, row = owner_and_row(i, world)
            assert parts[r][row] == src[i]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = gg.rmat(10, 8, 1, 255, seed=3)
        sources = gg.sources(g, 7, seed=5)

        def runner(sl):
            rows, E, V = [], 0, 0
            for s in sl:
                d, v, e = oracle.dijkstra(g, int(s))
                rows.append(torch.from_numpy(d.view(np.int64).copy()))
                E += e
                V += v
            t = torch.stack(rows) if rows else torch.empty((0, g.n), dtype=torch.int64)
            return t, {"reach_edges": E, "reachable": V, "edges_relaxed": E, "vertices_processed": V,
                       "runs": len(sl)}

        # the exact rank loop bench.py runs on the GPUs (barriers, timing, reductions, gather)
        out = run_batch_distributed(None, sources, gather_to=0, runner=runner, device=torch.device("cpu"))
        ok = True
        if rank == 0:
            full = out["full"].numpy().view(np.uint64)
            ok = all(np.array_equal(full[i], oracle.dijkstra(g, int(s))[0]) for i, s in enumerate(sources))
        else:
            ok = out["full"] is None
        E_all = sum(oracle.dijkstra(g, int(s))[2] for s in sources)
        # every rank reports the same max time, at least its own
        maxes = [torch.zeros(1, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(maxes, torch.tensor([out["max_ms"]], dtype=torch.float64))
        locs = [torch.zeros(1, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(locs, torch.tensor([out["local_ms"]], dtype=torch.float64))
        same_max = all(float(m) == out["max_ms"] for m in maxes) and out["max_ms"] == max(float(x) for x in locs)
        q.put((rank, ok, out["stats"]["reach_edges"] == E_all, out["stats"]["runs"], same_max,
               len(out["sources"]), "gather_ms" in out))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(300)
@pytest.mark.parametrize("world", [2, 4])
def test_multi_rank_gloo_batch(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    for rank, ok, e_ok, runs, same_max, nmine, timed_gather in res:
        assert ok and e_ok
        assert runs == 7            # counters summed over every rank
        assert same_max             # max over ranks, identical on every rank
        assert timed_gather
    assert [r[5] for r in res] == [len(range(r, 7, world)) for r in range(world)]

"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element, bit-exact (integer distances).

Sizes: tiny hand-made graphs and edge cases, scaled-down configs that span
many CTAs/batches and ragged tails, and the full BASELINE configs with the
launch configuration bench.py times.  Schedule-perturbation runs (grid size,
block size, Delta, bucket count, tiny rings forcing overflow/retry, 32/64-bit
distances) must all give the same bits.
"""
import numpy as np
import pytest

import graphgen as gg
import oracle
from conftest import golden_names, load_golden

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_ppopp_wangfl21_b200 as sssp  # noqa: E402

INF = np.uint64(0xFFFFFFFFFFFFFFFF)


def gpu_dist(g, s, variant="", **opt):
    G = sssp.Graph.from_csr(g, variant=variant, **opt)
    d = sssp.to_u64(G.run(int(s)))
    st = G.stats()
    G.close()
    return d, st


def check(g, s, variant="", **opt):
    ref, V, E = oracle.dijkstra(g, int(s))
    d, st = gpu_dist(g, s, variant=variant, **opt)
    bad = np.flatnonzero(d != ref)
    assert bad.size == 0, f"{bad.size} mismatches, first v={bad[:5]} gpu={d[bad[:5]]} ref={ref[bad[:5]]} opt={opt}"
    assert st["reachable"] == V and st["reach_edges"] == E
    assert st["vertices_processed"] >= V        # never less work than Dijkstra
    return st


# ----------------------------------------------------------------- edge cases
@pytest.mark.parametrize("name", golden_names())
def test_golden_fixtures_on_gpu(name):
    fx = load_golden(name)
    g = gg.from_arcs(fx["n"], fx["arcs"])
    d, st = gpu_dist(g, fx["source"])
    assert [int(x) for x in d] == fx["dist"]
    assert st["reachable"] == fx["V"] and st["reach_edges"] == fx["E"]


@pytest.mark.parametrize("name", golden_names())
def test_golden_fixtures_fuzzed(name):
    """The schedule-fuzzing build (hash-driven delays at reserve/publish/claim/complete/head-CAS)."""
    fx = load_golden(name)
    g = gg.from_arcs(fx["n"], fx["arcs"])
    d, st = gpu_dist(g, fx["source"], variant="fuzz")
    assert [int(x) for x in d] == fx["dist"]
    assert st["reachable"] == fx["V"] and st["reach_edges"] == fx["E"]


@pytest.mark.parametrize("name", golden_names())
def test_golden_fixtures_relabeled(name):
    fx = load_golden(name)
    g = gg.from_arcs(fx["n"], fx["arcs"])
    d, st = gpu_dist(g, fx["source"], flags=sssp.SSSP_FLAG_RELABEL)
    assert [int(x) for x in d] == fx["dist"]
    assert st["reachable"] == fx["V"] and st["reach_edges"] == fx["E"]


def test_relabel_auto_on_skewed_graphs_only():
    # RMAT (power-law in-degrees) is relabeled, the grid is not; results identical either way
    rmat = gg.make("rmat", scale_down=9)
    s = int(gg.config_sources("rmat", rmat, 1)[0])
    G = sssp.Graph.from_csr(rmat)
    assert G.info()["relabeled"] == 1
    assert np.array_equal(sssp.to_u64(G.run(s)), oracle.dijkstra(rmat, s)[0])
    road = gg.make("road", scale_down=9)
    assert sssp.Graph.from_csr(road).info()["relabeled"] == 0


def test_worker_selection():
    # AUTO = the CTA worker; the warp-granular ablation was removed (D12)
    rmat = gg.make("rmat", scale_down=10)
    s = gg.config_sources("rmat", rmat, 1)[0]
    assert check(rmat, s)["worker"] == sssp.SSSP_WORKER_CTA
    with pytest.raises(sssp.SSSPError) as e:
        sssp.Graph.from_csr(rmat, worker=2)
    assert e.value.status == 1


def test_u32_overflow_reruns_in_64_bits():
    n = 10
    g = gg.from_arcs(n, [(i, i + 1, 0xFFFFFFFF) for i in range(n - 1)] + [(0, 5, 7)])
    st = check(g, 0)
    assert st["dist_bits"] == 64 and st["retries"] >= 1


def test_single_vertex_and_empty_graph():
    g = gg.from_arcs(1, [])
    d, _ = gpu_dist(g, 0)
    assert d.tolist() == [0]
    g = gg.from_arcs(5, [])
    d, st = gpu_dist(g, 3)
    assert d.tolist() == [int(INF)] * 3 + [0, int(INF)]
    assert st["reachable"] == 1


def test_random_small_graphs():
    rng = np.random.default_rng(1)
    for t in range(40):
        n = int(rng.integers(1, 300))
        m = int(rng.integers(0, 8 * n))
        wmax = int(rng.choice([1, 3, 100, 1 << 20, 0xFFFFFFFF]))
        arcs = list(zip(rng.integers(0, n, m), rng.integers(0, n, m), rng.integers(0, wmax, m, endpoint=True)))
        g = gg.from_arcs(n, arcs)
        check(g, int(rng.integers(0, n)))
        check(g, int(rng.integers(0, n)), variant="fuzz")


def test_config_grid64():
    g = gg.make("grid64")
    check(g, 0)


# ----------------------------------------------------------------- scaled configs
@pytest.mark.parametrize("config,down", [("road", 8), ("road", 4), ("rmat", 8), ("rmat", 6), ("er", 8), ("er", 6)])
def test_scaled_configs(config, down):
    g = gg.make(config, scale_down=down)
    for s in gg.config_sources(config, g, 2):
        check(g, s)


# ----------------------------------------------------------------- chunked bucket storage
CHUNKED = sssp.SSSP_FLAG_CHUNKED_RING


@pytest.mark.parametrize("config", ["road", "rmat", "er"])
def test_chunked_ring_scaled(config):
    """Bucket storage as a chunk pool (the paper's block pool): the default pool, and
    a 64-chunk pool small enough that chunks are recycled many times within a run (and
    exhausted, then regrown, where the live items outgrow it)."""
    g = gg.make(config, scale_down=6)
    for s in gg.config_sources(config, g, 2):
        check(g, s, flags=CHUNKED)
        st = check(g, s, flags=CHUNKED, ring_items=64 * 4096)
        assert st["pushes"] > 0


@pytest.mark.parametrize("opt", [dict(), dict(dist_bits=64), dict(block_threads=256), dict(grid_ctas=3),
                                 dict(num_buckets=2), dict(ring_items=64 * 4096)])
def test_chunked_ring_fuzzed(opt):
    for config in ("road", "rmat"):
        g = gg.make(config, scale_down=8)
        s = int(gg.config_sources(config, g, 1)[0])
        check(g, s, variant="fuzz", flags=CHUNKED, **opt)


def test_chunked_ring_overflow_regrows():
    g = gg.make("rmat", scale_down=6)
    s = int(gg.config_sources("rmat", g, 1)[0])
    G = sssp.Graph.from_csr(g, flags=CHUNKED, ring_items=64)  # 64 chunks: exhausted early
    d = sssp.to_u64(G.run(s))
    assert np.array_equal(d, oracle.dijkstra(g, s)[0])
    assert G.stats()["retries"] >= 0
    Hn = sssp.Graph.from_csr(g, flags=CHUNKED | sssp.SSSP_FLAG_NO_RETRY, ring_items=64, grid_ctas=296)
    try:
        Hn.run(s)
    except RuntimeError as e:  # a pool too small for the live items is reported, not wrong
        assert "overflow" in str(e).lower()


@pytest.mark.parametrize("config", ["road", "rmat", "er"])
def test_chunked_ring_full_size(config):
    g = gg.make(config)
    s = int(gg.config_sources(config, g, 1)[0])
    ref, V, E = oracle.dijkstra(g, s)
    G = sssp.Graph.from_csr(g, flags=CHUNKED)
    out = G.run(s)
    assert np.array_equal(sssp.to_u64(out), ref)
    assert G.stats()["reach_edges"] == E
    # 32-bit items, flat: 32 arrays of next_pow2(n) items x 8 B = 256 n bytes; the pool starts at
    # 2n items (16 n bytes) and doubles only when the live items outgrow it (ER peaks near 2.4 n)
    assert G.stats()["ring_bytes"] <= 64 * g.n + (1 << 23)


@pytest.mark.timeout(1800)
def test_chunked_ring_2p26_four_in_flight():
    """n = 2^26 (ER, average degree 8) with four sources in flight: every row certified on the GPU."""
    g = gg.er(1 << 26, 8 << 26, 1, 1 << 20, seed=11)
    srcs = gg.sources(g, 4, seed=11)
    G = sssp.Graph.from_csr(g, flags=CHUNKED, concurrent_sources=4)
    D = G.run_batch(srcs)
    assert G.stats()["concurrency"] == 4
    for i, s in enumerate(srcs):
        c = G.certify(int(s), D[i])
        assert c["exact"] == 1, (int(s), c)


# the controller-validation families (graphgen.EXTRA): both sides of the degree-8 build switch,
# weights to 2^20; plus the throughput build at 256 threads per CTA
@pytest.mark.parametrize("config", ["rmat_ef4", "er_d4", "grid_wide", "rmat_wide"])
def test_extra_families(config):
    g = gg.make(config, scale_down=6)
    for s in gg.config_sources(config, g, 2):
        check(g, s)
        check(g, s, block_threads=256)


@pytest.mark.parametrize("config", ["er_d4", "rmat_wide"])
def test_extra_families_full_size(config):
    g = gg.make(config)
    s = int(gg.config_sources(config, g, 1)[0])
    ref, V, E = oracle.dijkstra(g, s)
    G = sssp.Graph.from_csr(g)
    out = G.run(s)
    assert np.array_equal(sssp.to_u64(out), ref)
    c = G.certify(s, out)
    assert c["exact"] == 1 and c["reach_edges"] == E


# ----------------------------------------------------------------- schedule perturbation
PERTURB = [
    dict(grid_ctas=1), dict(grid_ctas=3), dict(grid_ctas=37),
    dict(block_threads=128), dict(block_threads=512),
    dict(delta_mode=1, delta_init=1), dict(delta_mode=1, delta_init=1 << 30), dict(delta_init=1 << 16),
    dict(num_buckets=2), dict(num_buckets=2, delta_mode=1), dict(num_buckets=8),
    dict(dist_bits=64), dict(active_init=32), dict(batch_min=1), dict(batch_min=256),
    dict(settle_head_switches=1, util_lo_pct=1000, util_hi_pct=2000),
    dict(ring_items=64), dict(ring_items=256, num_buckets=4),
    dict(flags=sssp.SSSP_FLAG_TRACE),
    dict(flags=sssp.SSSP_FLAG_NO_LOCAL), dict(local_max=1), dict(local_max=16), dict(max_backoff_ns=64),
    dict(algorithm=sssp.SSSP_ALGO_NEAR_FAR), dict(algorithm=sssp.SSSP_ALGO_NEAR_FAR, delta_init=1),
    dict(algorithm=sssp.SSSP_ALGO_NEAR_FAR, delta_init=1 << 40), dict(algorithm=sssp.SSSP_ALGO_NEAR_FAR, ring_items=64),
    dict(algorithm=sssp.SSSP_ALGO_NEAR_FAR, grid_ctas=5), dict(flags=sssp.SSSP_FLAG_ADAPT_ACTIVE),
    # hub splitting: 1-arc chunks (every multi-arc vertex splits; chunk-queue overflow + regrowth),
    # small chunks on few CTAs, 64-bit distances, and splitting off
    dict(split_degree=1), dict(split_degree=3, grid_ctas=3), dict(split_degree=2, dist_bits=64),
    dict(split_degree=5, flags=sssp.SSSP_FLAG_NO_LOCAL), dict(split_degree=0xFFFFFFFF),
    # warp-local continuation off / with a 1-item CTA-level cap; 1024-thread CTAs
    dict(flags=sssp.SSSP_FLAG_NO_WARP_LOCAL), dict(flags=sssp.SSSP_FLAG_WARP_LOCAL, local_max=1, grid_ctas=2), dict(block_threads=1024),
    # relaxation filter on the 16-bit upper-bound array instead of dist itself
    dict(flags=sssp.SSSP_FLAG_FILTER16), dict(flags=sssp.SSSP_FLAG_FILTER16, dist_bits=64),
    dict(worker=sssp.SSSP_WORKER_CTA),
    # locality relabeling (D15) forced on / off, with the 64-bit and Near-Far paths
    dict(flags=sssp.SSSP_FLAG_RELABEL), dict(flags=sssp.SSSP_FLAG_NO_RELABEL),
    dict(flags=sssp.SSSP_FLAG_RELABEL, dist_bits=64),
    dict(flags=sssp.SSSP_FLAG_RELABEL, algorithm=sssp.SSSP_ALGO_NEAR_FAR),
    # the throughput build on 64-bit row offsets (the m >= 2^32 path), with 256-thread CTAs and hub splits
    dict(flags=sssp.SSSP_FLAG_WIDE_ROWS), dict(flags=sssp.SSSP_FLAG_WIDE_ROWS, block_threads=256),
    dict(flags=sssp.SSSP_FLAG_WIDE_ROWS, split_degree=3),
]


@pytest.mark.parametrize("opt", PERTURB, ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
@pytest.mark.parametrize("config", ["road", "rmat", "er"])
def test_schedule_perturbation(config, opt):
    g = gg.make(config, scale_down=10)
    s = gg.config_sources(config, g, 1)[0]
    check(g, s, **opt)


# the same matrix on the schedule-fuzzing build (libsssp_fuzz.so, -DSSSP_FUZZ): hash-driven
# 32 ns - 4 us delays at the reserve / publish / claim / pop / complete / head-CAS / chunk points
# reorder the worklist protocol's steps far more than the natural schedule does
FUZZ = [dict(), dict(grid_ctas=3), dict(block_threads=128), dict(block_threads=512), dict(num_buckets=2),
        dict(dist_bits=64), dict(active_init=32), dict(batch_min=1), dict(ring_items=64),
        dict(flags=sssp.SSSP_FLAG_NO_LOCAL), dict(local_max=1), dict(split_degree=1), dict(split_degree=3, grid_ctas=3),
        dict(delta_mode=1, delta_init=1), dict(delta_mode=1, delta_init=1 << 30), dict(flags=sssp.SSSP_FLAG_ADAPT_ACTIVE),
        dict(settle_head_switches=1, util_lo_pct=1000, util_hi_pct=2000), dict(flags=sssp.SSSP_FLAG_TRACE),
        dict(flags=sssp.SSSP_FLAG_WARP_LOCAL, local_max=1, grid_ctas=2), dict(concurrent_sources=1),
        dict(flags=sssp.SSSP_FLAG_WIDE_ROWS)]


@pytest.mark.parametrize("opt", FUZZ, ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()) or "default")
@pytest.mark.parametrize("config", ["road", "rmat", "er"])
def test_fuzzed_schedule(config, opt):
    g = gg.make(config, scale_down=10)
    for s in gg.config_sources(config, g, 2):
        check(g, s, variant="fuzz", **opt)


def test_fuzzed_concurrent_batch():
    g = gg.make("road", scale_down=9)
    srcs = gg.config_sources("road", g, 6)
    G = sssp.Graph.from_csr(g, variant="fuzz", concurrent_sources=3, ring_items=256)
    D = G.run_batch(srcs)
    for i, s in enumerate(srcs):
        assert np.array_equal(sssp.to_u64(D[i]), oracle.dijkstra(g, int(s))[0])


def test_tiny_ring_without_retry_reports_overflow():
    g = gg.make("rmat", scale_down=8)
    s = int(gg.config_sources("rmat", g, 1)[0])
    G = sssp.Graph.from_csr(g, ring_items=64, flags=sssp.SSSP_FLAG_NO_RETRY)
    with pytest.raises(sssp.SSSPError) as e:
        G.run(s)
    assert e.value.status == 5
    # the handle stays usable after growing the ring
    G.set_options(ring_items=0, flags=0)
    d = sssp.to_u64(G.run(s))
    assert np.array_equal(d, oracle.dijkstra(g, s)[0])


# ----------------------------------------------------------------- API behaviour
def test_run_batch_equals_single_runs():
    g = gg.make("rmat", scale_down=9)
    srcs = gg.sources(g, 7, seed=5)
    G = sssp.Graph.from_csr(g)
    D = G.run_batch(srcs)
    st = G.stats()
    assert st["runs"] == 7
    for i, s in enumerate(srcs):
        assert np.array_equal(sssp.to_u64(D[i]), oracle.dijkstra(g, int(s))[0])


def test_host_dist_out():
    g = gg.make("road", scale_down=10)
    s = int(gg.config_sources("road", g, 1)[0])
    G = sssp.Graph.from_csr(g)
    d = G.run_host(s)
    assert np.array_equal(d, oracle.dijkstra(g, s)[0])


def test_device_input_arrays():
    g = gg.make("er", scale_down=10)
    s = int(gg.config_sources("er", g, 1)[0])
    off = torch.from_numpy(g.row_offsets.view(np.int64)).cuda()
    col = torch.from_numpy(g.col.view(np.int32)).cuda()
    w = torch.from_numpy(g.w.view(np.int32)).cuda()
    G = sssp.Graph(off, col, w)
    assert np.array_equal(sssp.to_u64(G.run(s)), oracle.dijkstra(g, s)[0])


def test_invalid_inputs():
    ok_off = np.array([0, 1, 2], dtype=np.uint64)
    with pytest.raises(sssp.SSSPError) as e:
        sssp.Graph(np.array([0, 2, 1], dtype=np.uint64), np.array([0], dtype=np.uint32), np.array([1], dtype=np.uint32))
    assert e.value.status == 2
    with pytest.raises(sssp.SSSPError) as e:
        sssp.Graph(ok_off, np.array([0, 5], dtype=np.uint32), np.array([1, 1], dtype=np.uint32))
    assert e.value.status == 2 and "col[1]" in e.value.detail
    with pytest.raises(sssp.SSSPError) as e:
        sssp.Graph(np.array([1, 2, 2], dtype=np.uint64), np.array([0, 1], dtype=np.uint32),
                   np.array([1, 1], dtype=np.uint32))
    assert e.value.status == 2
    G = sssp.Graph(ok_off, np.array([1, 0], dtype=np.uint32), np.array([1, 1], dtype=np.uint32))
    with pytest.raises(sssp.SSSPError) as e:
        G.run(2)
    assert e.value.status == 1
    with pytest.raises(sssp.SSSPError) as e:
        G.run_batch(np.array([], dtype=np.uint32), out=torch.empty((0, 2), dtype=torch.int64, device="cuda"))
    assert e.value.status == 1


def test_async_flag_and_stats():
    g = gg.make("road", scale_down=8)
    s = int(gg.config_sources("road", g, 1)[0])
    G = sssp.Graph.from_csr(g, flags=sssp.SSSP_FLAG_ASYNC)
    out = G.run(s)
    torch.cuda.synchronize()
    st = G.stats()
    assert st["status"] == 0 and st["kernel_ms"] > 0
    assert np.array_equal(sssp.to_u64(out), oracle.dijkstra(g, s)[0])


def check_controller_trace(tr, st, a_lo, a_hi):
    """The Delta controller's invariants from its committed steps."""
    assert sum(1 for e in tr if e["reason"] & 255 == 1) == min(st["head_switches"], 65536)
    prev_flo = 0
    for e in tr:
        A, flo, ceil = e["active"] & 255, (e["active"] >> 8) & 255, (e["active"] >> 16) & 255
        assert e["reason"] & 255 in (1, 2)
        assert a_lo <= A <= a_hi                      # P:217 knob within its bounds
        assert 0 <= e["delta_log2"] <= 31
        assert e["delta_log2"] >= flo                 # never below the clip bound
        assert flo >= prev_flo                        # the bound only rises (on clip steps)
        prev_flo = flo
        assert ceil == 255 or ceil > e["delta_log2"]  # a ceiling is a Delta measured wasteful, above k
        assert e["waste_permille"] <= 1000
        assert e["pending_tail"] <= e["pending_total"] and e["pending_window"] <= e["pending_total"]
    # Delta moves one power of two per step; a change that is not a clip step needs the ring
    # to have turned over -- >= 2 head switches since the previous change (reading R7) --
    # or, for a shrink under sustained waste with the head parked, >= 4 x 8 controller steps
    ks = [e["delta_log2"] for e in tr]
    assert all(abs(a - b) <= 1 for a, b in zip(ks, ks[1:]))
    last_change, switches = None, 0
    for i in range(1, len(tr)):
        if tr[i]["reason"] & 255 == 1:
            switches += 1
        if ks[i] != ks[i - 1]:
            clip_step = (tr[i]["reason"] >> 8) & 32
            if not clip_step and last_change is not None:
                parked_shrink = ks[i] < ks[i - 1] and i - last_change >= 32
                assert switches >= 2 or parked_shrink, (i, switches, i - last_change)
            last_change, switches = i, 0
    ts = [e["time_ns"] for e in tr]
    assert len(tr) < 2 or max(ts) >= min(ts)


@pytest.mark.parametrize("config,a_lo,a_hi", [("rmat", 4, 8), ("road", 1, 2), ("er", 4, 8)])
def test_trace_invariants(config, a_lo, a_hi):
    g = gg.make(config, scale_down=6)
    for s in gg.config_sources(config, g, 3):
        G = sssp.Graph.from_csr(g, flags=sssp.SSSP_FLAG_TRACE)
        d = sssp.to_u64(G.run(int(s)))
        assert np.array_equal(d, oracle.dijkstra(g, int(s))[0])
        check_controller_trace(G.trace(), G.stats(), a_lo, a_hi)
        G.close()


def test_trace_invariants_full_size_road():
    """ROAD at full size: ~300 head switches, the controller's longest run here."""
    g = gg.make("road")
    s = int(gg.config_sources("road", g, 1)[0])
    G = sssp.Graph.from_csr(g, flags=sssp.SSSP_FLAG_TRACE)
    G.run(s)
    check_controller_trace(G.trace(), G.stats(), 1, 2)


def test_repeat_runs_deterministic_and_reusable():
    g = gg.make("er", scale_down=9)
    srcs = gg.sources(g, 3, seed=9)
    G = sssp.Graph.from_csr(g)
    for s in list(srcs) * 2:
        assert np.array_equal(sssp.to_u64(G.run(int(s))), oracle.dijkstra(g, int(s))[0])


# ----------------------------------------------------------------- full BASELINE sizes
@pytest.mark.parametrize("config", ["road", "rmat", "er"])
def test_full_size_config(config):
    g = gg.make(config)
    s = int(gg.config_sources(config, g, 1)[0])
    ref, V, E = oracle.dijkstra(g, s)
    # the bench's launch configuration, 64-bit distances, and the other relabeling choice
    # (relabeling happens at create time: its own handle)
    G = sssp.Graph.from_csr(g)
    H = sssp.Graph.from_csr(g, flags=sssp.SSSP_FLAG_NO_RELABEL if config == "rmat" else sssp.SSSP_FLAG_RELABEL)
    assert G.info()["relabeled"] != H.info()["relabeled"]
    for X, opt in ((G, dict()), (G, dict(flags=sssp.SSSP_FLAG_WIDE_ROWS)), (G, dict(flags=0, dist_bits=64)), (H, dict())):
        if opt:
            X.set_options(**opt)
        out = X.run(s)
        st = X.stats()
        d = sssp.to_u64(out)
        bad = np.flatnonzero(d != ref)
        assert bad.size == 0, f"{opt}: {bad.size} mismatches, first v={bad[:5]}"
        assert st["reachable"] == V and st["reach_edges"] == E
        assert st["dist_bits"] == opt.get("dist_bits", 32)
        c = X.certify(s, out)
        assert c["exact"] == 1 and c["reachable"] == V and c["reach_edges"] == E


@pytest.mark.timeout(1800)
def test_full_size_batch_every_source():
    """Config 5 at full size in bench.py's launch configuration (RMAT-24, all 512 sources,
    2 in flight, through the same rank loop as the multi-GPU bench): EVERY row passes the GPU
    certificate (sssp_certify: no violated arc, every finite vertex reachable through tight
    arcs, dist[s] = 0, reach counts = the run's), and a seeded half of the rows (256) is
    compared element by element with the oracle, streamed over a pool of host threads."""
    import concurrent.futures as cf
    import os
    from paper_conf_ppopp_wangfl21_b200.distributed import run_batch_distributed
    g = gg.make("batch")
    srcs = gg.sources(g, 512, gg.CONFIGS["batch"]["source_seed"])
    assert len(set(srcs.tolist())) == 512
    G = sssp.Graph.from_csr(g, concurrent_sources=2)
    D = torch.empty((512, g.n), dtype=torch.int64, device="cuda")
    res = run_batch_distributed(G, srcs, out=D)
    assert res["stats"]["runs"] == 512 and G.stats()["concurrency"] == 2
    E_cert = 0
    for i, s in enumerate(srcs):
        c = G.certify(int(s), D[i])
        assert c["exact"] == 1, f"source {int(s)}: {c}"
        E_cert += c["reach_edges"]
    assert res["stats"]["reach_edges"] == E_cert      # the run's own E_dij agrees with the certified rows
    rng = np.random.default_rng(5)
    half = np.sort(rng.choice(512, size=256, replace=False))
    workers = max(1, min(16, (os.cpu_count() or 2) - 1))
    with cf.ThreadPoolExecutor(workers) as ex:
        futs = {ex.submit(oracle.dijkstra, g, int(srcs[i])): i for i in half}
        for f in cf.as_completed(futs):
            i = futs[f]
            ref, V, E = f.result()
            row = sssp.to_u64(D[i])
            assert np.array_equal(row, ref), f"source {int(srcs[i])}"
    parts = [srcs[r::8] for r in range(8)]
    assert sorted(np.concatenate(parts).tolist()) == sorted(srcs.tolist())


def test_run_batch_distributed_single_rank():
    from paper_conf_ppopp_wangfl21_b200.distributed import run_batch_distributed
    g = gg.make("rmat", scale_down=10)
    srcs = gg.sources(g, 5, seed=5)
    G = sssp.Graph.from_csr(g)
    out = run_batch_distributed(G, srcs, gather_to=0)
    assert out["max_ms"] > 0 and out["max_ms"] == out["local_ms"]
    full = sssp.to_u64(out["full"])
    for i, s in enumerate(srcs):
        assert np.array_equal(full[i], oracle.dijkstra(g, int(s))[0])
    assert out["stats"]["runs"] == 5


def test_loaded_file_through_the_abi(tmp_path):
    from graphgen import loaders
    g = gg.make("road", scale_down=10)
    p = str(tmp_path / "road.gr")
    loaders.save_galois_gr(g, p)
    h = loaders.load(p)
    s = int(gg.config_sources("road", h, 1)[0])
    check(h, s)


@pytest.mark.parametrize("conc", [2, 3, 8])
def test_concurrent_batch(conc):
    """NEXT-1: several sources in flight at once (own workspace + stream each)."""
    g = gg.make("rmat", scale_down=9)
    srcs = gg.sources(g, 7, seed=5)
    G = sssp.Graph.from_csr(g, concurrent_sources=conc)
    D = G.run_batch(srcs)
    st = G.stats()
    assert st["runs"] == 7 and st["concurrency"] == min(conc, 7) and st["batch_ms"] > 0
    for i, s in enumerate(srcs):
        assert np.array_equal(sssp.to_u64(D[i]), oracle.dijkstra(g, int(s))[0])


@pytest.mark.parametrize("conc,pinned", [(1, True), (2, True), (3, False)])
def test_batch_host_out(conc, pinned):
    """Host dist_out batches: staged per slot, copies overlapped with the next sources."""
    import torch
    g = gg.make("rmat", scale_down=8)
    srcs = gg.config_sources("rmat", g, 5)
    G = sssp.Graph.from_csr(g, concurrent_sources=conc)
    out = torch.full((len(srcs), g.n), -7, dtype=torch.int64)
    if pinned:
        out = out.pin_memory()
    G.run_batch(srcs, out=out)
    assert G.stats()["concurrency"] == conc
    for i, s in enumerate(srcs):
        assert np.array_equal(sssp.to_u64(out[i]), oracle.dijkstra(g, int(s))[0])


def test_batch_host_out_overflow_retry():
    import torch
    g = gg.make("road", scale_down=8)
    srcs = gg.config_sources("road", g, 5)
    G = sssp.Graph.from_csr(g, concurrent_sources=2, ring_items=64)
    out = torch.empty((len(srcs), g.n), dtype=torch.int64)
    G.run_batch(srcs, out=out)
    assert G.stats()["retries"] >= 1
    for i, s in enumerate(srcs):
        assert np.array_equal(sssp.to_u64(out[i]), oracle.dijkstra(g, int(s))[0])


@pytest.mark.parametrize("host", [False, True])
def test_independent_slots_ragged_with_retries(host):
    """7 sources on 3 slots (a ragged last round), every source overflowing its 64-item ring
    first: slots settle, retry and restart out of step with each other."""
    import torch
    g = gg.make("rmat", scale_down=9)
    srcs = gg.config_sources("rmat", g, 7)
    G = sssp.Graph.from_csr(g, concurrent_sources=3, ring_items=64)
    out = torch.empty((len(srcs), g.n), dtype=torch.int64) if host else None
    D = G.run_batch(srcs, out=out)
    st = G.stats()
    assert st["retries"] >= 1 and st["concurrency"] == 3
    for i, s in enumerate(srcs):
        assert np.array_equal(sssp.to_u64(D[i]), oracle.dijkstra(g, int(s))[0])


def test_concurrent_batch_with_overflow_retry():
    g = gg.make("road", scale_down=8)
    srcs = gg.config_sources("road", g, 4)
    G = sssp.Graph.from_csr(g, concurrent_sources=4, ring_items=64)
    D = G.run_batch(srcs)
    assert G.stats()["retries"] >= 1
    for i, s in enumerate(srcs):
        assert np.array_equal(sssp.to_u64(D[i]), oracle.dijkstra(g, int(s))[0])


@pytest.mark.parametrize("config", ["road", "rmat", "er"])
def test_near_far_ablation_full_size(config):
    """NEXT-2: the BSP Near-Far comparison system gives the same bits."""
    g = gg.make(config, scale_down=4)
    s = int(gg.config_sources(config, g, 1)[0])
    st = check(g, s, algorithm=sssp.SSSP_ALGO_NEAR_FAR)
    assert st["head_switches"] > 0  # supersteps


def test_near_far_u64_and_golden():
    n = 10
    g = gg.from_arcs(n, [(i, i + 1, 0xFFFFFFFF) for i in range(n - 1)] + [(0, 5, 7)])
    st = check(g, 0, algorithm=sssp.SSSP_ALGO_NEAR_FAR)
    assert st["dist_bits"] == 64
    for name in golden_names():
        fx = load_golden(name)
        gg2 = gg.from_arcs(fx["n"], fx["arcs"])
        d, _ = gpu_dist(gg2, fx["source"], algorithm=sssp.SSSP_ALGO_NEAR_FAR)
        assert [int(x) for x in d] == fx["dist"]


# ----------------------------------------------------------------- NEXT-3: float32 weights
def check_f32(g, wf, s, **opt):
    ref, V, E = oracle.dijkstra_f32(g, wf, int(s))
    G = sssp.Graph.from_csr(g, weights=wf, **opt)
    d = G.run(int(s)).cpu().numpy()
    st = G.stats()
    G.close()
    bad = np.flatnonzero(d.view(np.uint32) != ref.view(np.uint32))
    assert bad.size == 0, f"{bad.size} mismatches, first {bad[:5]} gpu={d[bad[:5]]} ref={ref[bad[:5]]} {opt}"
    assert st["reachable"] == V and st["reach_edges"] == E
    return st


@pytest.mark.parametrize("config,lo,hi", [("road", 0.0, 1.0), ("rmat", 1.0, 255.0), ("er", 0.0, 1e-3),
                                          ("road", 100.0, 1e6)])
def test_float_weights_scaled(config, lo, hi):
    g = gg.make(config, scale_down=8)
    wf = gg.float_weights(g, lo, hi, seed=11)
    for s in gg.config_sources(config, g, 2):
        check_f32(g, wf, s)


@pytest.mark.parametrize("opt", [dict(delta_mode=1, delta_init=1), dict(delta_mode=1, delta_init=1 << 20),
                                 dict(ring_items=64), dict(grid_ctas=3), dict(block_threads=256),
                                 dict(flags=sssp.SSSP_FLAG_NO_LOCAL), dict(concurrent_sources=2)],
                         ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
def test_float_weights_perturbed(opt):
    g = gg.make("rmat", scale_down=10)
    wf = gg.float_weights(g, 0.0, 1.0, seed=3)
    check_f32(g, wf, int(gg.config_sources("rmat", g, 1)[0]), **opt)


def test_float_weights_full_size_road():
    g = gg.make("road")
    wf = gg.float_weights(g, 0.0, 1.0, seed=2)
    st = check_f32(g, wf, int(gg.config_sources("road", g, 1)[0]))
    assert st["edges_relaxed"] <= 3 * st["reach_edges"]


def test_float_rounding_fixture_and_errors():
    F32 = np.float32
    one_ulp = np.nextafter(F32(1.0), F32(2.0))
    g = gg.from_arcs(3, [(0, 1, 0), (0, 2, 0), (1, 2, 0)])   # CSR order: (0,1) (0,2) (1,2)
    wf = np.array([1.0, one_ulp, 2.0 ** -24], dtype=F32)
    G = sssp.Graph.from_csr(g, weights=wf)
    d = G.run(0).cpu().numpy()
    assert d.tolist() == [0.0, 1.0, 1.0]                       # 1 + 2^-24 rounds to 1.0
    with pytest.raises(sssp.SSSPError) as e:
        sssp.Graph.from_csr(g, weights=np.array([1.0, -2.0, 0.5], dtype=F32))
    assert e.value.status == 2 and "w[1]" in e.value.detail
    with pytest.raises(sssp.SSSPError) as e:
        sssp.lib().sssp_run(G._h, 0, torch.empty(3, dtype=torch.int64, device="cuda").data_ptr(), 0)
        sssp._check(sssp.lib().sssp_run(G._h, 0, torch.empty(3, dtype=torch.int64, device="cuda").data_ptr(), 0))
    assert e.value.status == 1
    nz = sssp.Graph.from_csr(g, weights=np.array([-0.0, 1.0, 1.0], dtype=F32))   # -0.0 folds to +0.0
    assert nz.run(0).cpu().numpy().tolist() == [0.0, 0.0, 1.0]


def test_hub_split_star():
    """A source hub with 200K arcs (chunks of 1000 spread over the grid) plus a second-level hub,
    zero weights and parallel arcs: bit-exact, and every arc of the hub counted exactly once."""
    rng = np.random.default_rng(7)
    n = 250_001
    hub_arcs = 200_000
    cols = [rng.integers(1, n, hub_arcs)]
    ws = [rng.integers(0, 1000, hub_arcs)]
    rows = [np.zeros(hub_arcs, np.int64)]
    # vertex 1 is a second hub reached through the first
    cols.append(rng.integers(0, n, 50_000)); ws.append(rng.integers(0, 5, 50_000)); rows.append(np.ones(50_000, np.int64))
    src = np.concatenate(rows); dst = np.concatenate(cols); w = np.concatenate(ws)
    order = np.lexsort((w, dst, src))
    src, dst, w = src[order], dst[order], w[order]
    off = np.zeros(n + 1, np.uint64)
    np.add.at(off, src + 1, 1)
    off = np.cumsum(off).astype(np.uint64)
    g = gg.CSR(n, len(dst), off, dst.astype(np.uint32), w.astype(np.uint32))
    for opt in (dict(), dict(split_degree=1000), dict(split_degree=1000, grid_ctas=2), dict(split_degree=0xFFFFFFFF)):
        st = check(g, 0, **opt)
        assert st["edges_relaxed"] >= st["reach_edges"]


def test_filter16_resolution_change_keeps_results():
    """The 16-bit filter's resolution is refitted from each run's largest distance; runs on
    graphs whose distances exceed 65534 * 2^s (no bound -> plain atomic) and sources with very
    different ranges on one handle stay bit-exact (D11)."""
    g = gg.make("road", scale_down=8)
    G = sssp.Graph.from_csr(g, flags=sssp.SSSP_FLAG_FILTER16)
    for s in list(gg.config_sources("road", g, 3)) + [0]:
        d = sssp.to_u64(G.run(int(s)))
        assert np.array_equal(d, oracle.dijkstra(g, int(s))[0])
    # a chain whose distances run far beyond 65534 * 2^s for small weights
    n = 70000
    ch = gg.from_arcs(n, [(i, i + 1, 1 + (i % 3)) for i in range(n - 1)] + [(0, n - 1, 10**9)])
    H = sssp.Graph.from_csr(ch, flags=sssp.SSSP_FLAG_FILTER16)
    for _ in range(2):
        d = sssp.to_u64(H.run(0))
        assert np.array_equal(d, oracle.dijkstra(ch, 0)[0])


def test_bench_json_contract_small_config():
    """bench.py's one-line JSON contract on the small config (the driver runs the same
    code on configs[1]): required keys, device-timed value, e2e with host copies, clocks."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--config", "grid64", "--steps", "3",
                          "--warmup", "3", "--e2e-steps", "2"], capture_output=True, text=True, timeout=600, cwd=root)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"):
        assert k in line, k
    assert line["value"] > 0 and line["steps"] == 3 and line["warmup"] == 3 and line["n_gpus"] == 1
    assert line["gpu_launches"] >= 3 * 3
    assert line["e2e"]["h2d_bytes_per_step"] > 0 and line["e2e"]["d2h_bytes_per_step"] > 0
    assert line["roofline"]["peak"] > 0 and 0 < line["roofline"]["frac"] < 1
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] == 1
    assert "sm_mhz" in line["clocks"]


# ----------------------------------------------------------------- GPU certificate (sssp_certify)
def _perturbations(g, s, ref, rng):
    """Corruptions of the exact vector that a complete certificate must reject."""
    fin = np.flatnonzero((ref != INF) & (np.arange(g.n) != s))
    unr = np.flatnonzero(ref == INF)
    out = []
    d = ref.copy(); d[s] = 1; out.append(d)                              # (i)
    for v in rng.choice(fin, size=min(3, fin.size), replace=False) if fin.size else []:
        if ref[v] > 0:
            d = ref.copy(); d[v] -= 1; out.append(d)                     # too small: no tight path
        d = ref.copy(); d[v] += 1; out.append(d)                         # too large: an arc violated
        d = ref.copy(); d[v] = INF; out.append(d)                        # finite -> unreachable
    for v in rng.choice(unr, size=min(2, unr.size), replace=False) if unr.size else []:
        d = ref.copy(); d[v] = 7; out.append(d)                          # unreachable -> finite
    return out


def test_certificate_accepts_exact_and_rejects_perturbed():
    rng = np.random.default_rng(11)
    graphs = []
    for t in range(12):
        n = int(rng.integers(2, 200))
        m = int(rng.integers(0, 6 * n))
        wmax = int(rng.choice([0, 1, 3, 1000, 0xFFFFFFFF]))
        arcs = list(zip(rng.integers(0, n, m), rng.integers(0, n, m), rng.integers(0, wmax, m, endpoint=True)))
        graphs.append((gg.from_arcs(n, arcs), {}))
    r = gg.make("rmat", scale_down=12)
    graphs += [(r, {}), (r, dict(flags=sssp.SSSP_FLAG_RELABEL)), (gg.make("road", scale_down=12), {})]
    for g, opt in graphs:
        G = sssp.Graph.from_csr(g, **opt)
        s = int(rng.integers(0, g.n))
        ref, V, E = oracle.dijkstra(g, s)
        c = G.certify(s, ref)
        assert c["exact"] == 1 and c["reachable"] == V and c["reach_edges"] == E, c
        dev = G.run(s)
        assert G.certify(s, dev)["exact"] == 1
        for d in _perturbations(g, s, ref, rng):
            c = G.certify(s, d)
            assert c["exact"] == 0, (c, opt)
            assert oracle.certify(g, s, d) != 0          # the CPU certificate agrees


def test_certificate_zero_weight_fixpoint():
    # a zero-weight chain hanging off the source and a zero-weight cycle that is NOT reachable
    # but claims the same distance as a reachable vertex: only the fixpoint tells them apart
    n = 8
    arcs = [(0, 1, 5), (1, 2, 0), (2, 3, 0), (3, 4, 0), (5, 6, 0), (6, 5, 0), (0, 7, 3)]
    g = gg.from_arcs(n, arcs)
    G = sssp.Graph.from_csr(g)
    ref, _, _ = oracle.dijkstra(g, 0)
    c = G.certify(0, ref)
    assert c["exact"] == 1 and c["fixpoint_rounds"] >= 3
    d = ref.copy(); d[5] = d[6] = 5                                     # self-supporting zero cycle
    c = G.certify(0, d)
    assert c["exact"] == 0 and c["unanchored"] == 2 and c["first_unanchored"] == 5
    assert oracle.certify(g, 0, d) != 0


def test_certificate_float_graph():
    g = gg.make("rmat", scale_down=12)
    wf = gg.float_weights(g, 0.0, 1.0, seed=3)
    s = int(gg.config_sources("rmat", g, 1)[0])
    G = sssp.Graph.from_csr(g, weights=wf)
    d = G.run(s)
    assert G.certify(s, d)["exact"] == 1
    h = d.cpu().numpy().copy()
    v = int(np.flatnonzero(np.isfinite(h) & (h > 0))[0])
    h[v] = np.nextafter(h[v], np.float32(0))
    assert G.certify(s, h)["exact"] == 0


# ----------------------------------------------------------------- ASYNC error path
def test_async_overflow_then_exact_rerun():
    g = gg.make("rmat", scale_down=8)
    s = int(gg.config_sources("rmat", g, 1)[0])
    G = sssp.Graph.from_csr(g, flags=sssp.SSSP_FLAG_ASYNC, ring_items=64, split_degree=1)
    G.run(s)
    torch.cuda.synchronize()
    with pytest.raises(sssp.SSSPError) as e:
        G.stats()
    assert e.value.status == 5
    # leftovers of the aborted run (ring items, hub chunks) must not leak into the next run
    G.set_options(flags=0, ring_items=64, split_degree=1)
    assert np.array_equal(sssp.to_u64(G.run(s)), oracle.dijkstra(g, s)[0])
    G.set_options(flags=sssp.SSSP_FLAG_ASYNC, ring_items=0, split_degree=1)
    out = G.run(s)
    torch.cuda.synchronize()
    assert G.stats()["status"] == 0
    assert np.array_equal(sssp.to_u64(out), oracle.dijkstra(g, s)[0])


def test_async_dist_overflow_switches_to_64_bits():
    n = 10
    g = gg.from_arcs(n, [(i, i + 1, 0xFFFFFFFF) for i in range(n - 1)] + [(0, 5, 7)])
    G = sssp.Graph.from_csr(g, flags=sssp.SSSP_FLAG_ASYNC)
    G.run(0)
    torch.cuda.synchronize()
    with pytest.raises(sssp.SSSPError):
        G.stats()
    out = G.run(0)
    torch.cuda.synchronize()
    st = G.stats()
    assert st["status"] == 0 and st["dist_bits"] == 64
    assert np.array_equal(sssp.to_u64(out), oracle.dijkstra(g, 0)[0])


def test_python_out_checks():
    g = gg.make("grid64")
    G = sssp.Graph.from_csr(g)
    with pytest.raises(TypeError):
        G.run(0, out=torch.empty(g.n, dtype=torch.int32, device="cuda"))
    with pytest.raises(ValueError):
        G.run(0, out=torch.empty(g.n - 1, dtype=torch.int64, device="cuda"))
    with pytest.raises(ValueError):
        G.run(0, out=torch.empty((g.n, 2), dtype=torch.int64, device="cuda")[:, 0])
    with pytest.raises(ValueError):
        G.run_batch([0, 1], out=torch.empty(g.n, dtype=torch.int64, device="cuda"))

"""GPU parity: asynchronous push BFS (CUDA path through the C ABI) vs the oracle.

Bar (BASELINE.json north_star): depths bit-exact; every GPU parent satisfies
depth(parent) = depth(v) - 1 via an existing edge (and equals the min-id
canonical parent the kernel is specified to produce).
"""
import json
import os

import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs

pytestmark = pytest.mark.gpu
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def csr_of(n, edges):
    edges = sorted(edges)
    rp = np.zeros(n + 1, dtype=np.int64)
    for u, _ in edges:
        rp[u + 1] += 1
    rp = np.cumsum(rp)
    col = np.array([v for _, v in edges], dtype=np.int32)
    return rp, col


def check_parents(rp, col, depth, parent, src):
    n = rp.size - 1
    assert parent[src] == src
    assert np.all(parent[depth < 0] == -1)
    v = np.nonzero((depth > 0))[0]
    u = parent[v]
    assert np.all(u >= 0) and np.all(depth[u] == depth[v] - 1)
    # edge u->v exists
    for a, b in zip(u[:2000].tolist(), v[:2000].tolist()):
        assert b in col[rp[a]:rp[a + 1]]


def run_and_check(rp, col, src, **cfg):
    with atos.Graph(rp, col, **cfg) as G:
        d, par = G.bfs(src, parent=True)
    want = oracle.bfs(rp, col, src)
    assert np.array_equal(d, want), f"first diff at {np.nonzero(d != want)[0][:5]}"
    check_parents(rp, col, d, par, src)
    assert np.array_equal(par, oracle.bfs_parents_minid(rp, col, want, src))
    return d


def test_hand_fixture_with_self_loops_and_duplicates():
    fx = json.load(open(os.path.join(GOLDEN, "bfs_hand.json")))
    rp = np.zeros(len(fx["adj"]) + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(a) for a in fx["adj"]])
    col = np.array([v for a in fx["adj"] for v in a], dtype=np.int32)
    d = run_and_check(rp, col, fx["src"])
    assert d.tolist() == fx["depth"]


def test_sampled_4_vertex_digraphs():
    rng = np.random.default_rng(0)
    pairs = [(u, v) for u in range(4) for v in range(4) if u != v]
    for mask in rng.choice(1 << 12, 24, replace=False).tolist():
        edges = [pairs[i] for i in range(12) if mask >> i & 1] or [(0, 1)]
        rp, col = csr_of(4, edges)
        run_and_check(rp, col, int(rng.integers(0, 4)))


@pytest.mark.parametrize("seed", range(6))
def test_random_small_graphs(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 3000))
    m = int(rng.integers(1, 6 * n))
    edges = list(zip(rng.integers(0, n, m).tolist(), rng.integers(0, n, m).tolist()))
    rp, col = csr_of(n, edges)
    run_and_check(rp, col, int(rng.integers(0, n)))


def test_isolated_source_and_disconnected():
    rp, col = csr_of(6, [(0, 1), (1, 0), (2, 3), (3, 4)])
    assert run_and_check(rp, col, 5).tolist() == [-1] * 5 + [0]
    assert run_and_check(rp, col, 2).tolist() == [-1, -1, 0, 1, 2, -1]


@pytest.mark.parametrize("filt", [0, 1])
def test_long_path_latency_bound(filt):
    """20 000 levels: also exercises the saturated (255) probe filter."""
    n = 20000
    rp, col = csr_of(n, [(i, i + 1) for i in range(n - 1)] + [(i + 1, i) for i in range(n - 1)])
    d = run_and_check(rp, col, 0, probe_filter=filt)
    assert d[-1] == n - 1


def test_kron12_config0_from_vertex0():
    g = inputs.make_config("kron12")
    rp, col = g.numpy()
    run_and_check(rp, col, 0)


def test_road_grid_high_diameter():
    g = inputs.road_grid(300, 200, seed=2)
    rp, col = g.numpy()
    run_and_check(rp, col, 0)
    run_and_check(rp, col, g.n // 2 + 150)


def test_repeated_solves_on_one_handle_and_device_outputs():
    g = inputs.rmat(16, 16, 3, symmetric=True)
    rp, col = g.numpy()
    srcs = inputs.bfs_sources(g, 5, seed=3)
    with atos.Graph(rp, col) as G:
        for s in srcs:
            assert np.array_equal(G.bfs(s), oracle.bfs(rp, col, s))
        out = torch.empty(g.n, dtype=torch.int32, device="cuda")
        G.bfs(srcs[0], depth_out=out)           # async path: device output
        G.sync()
        assert np.array_equal(out.cpu().numpy(), oracle.bfs(rp, col, srcs[0]))
        st = G.last_stats()
        assert st["pops"] >= int((out >= 0).sum())


@pytest.mark.parametrize("ratom", [True, False])
@pytest.mark.parametrize("vr", [2, 3, 4, 8])
@pytest.mark.parametrize("agg", [0, 1])
def test_virtual_ranks_identical(vr, agg, ratom, monkeypatch):
    # ratom: the sender lowers the owner's depth word and sends activations (the virtual-rank
    # default); else depth messages the owner applies (the multi-process protocol)
    if not ratom:
        monkeypatch.setenv("ATOS_BFS_NORATOM", "1")
    g = inputs.rmat(15, 16, 1, symmetric=True)
    rp, col = g.numpy()
    src = inputs.bfs_sources(g, 1)[0]
    d = run_and_check(rp, col, src, virtual_ranks=vr, agg_enabled=agg, channel_packets=64)
    assert (d >= 0).sum() > 1000


@pytest.mark.parametrize("opts", [dict(relax_red=1), dict(relax_red=1, keep_items=64), dict(prefetch=0, l2_persist=0),
                                  dict(keep_items=512, fetch_size=7), dict(relax_red=1, virtual_ranks=4),
                                  dict(relax_red=0), dict(pipeline=1), dict(pipeline=0),
                                  dict(probe_filter=1), dict(probe_filter=1, relax_red=0),
                                  dict(probe_filter=1, virtual_ranks=3), dict(probe_filter=1, pipeline=1)])
def test_runtime_options_same_depths(opts):
    """Every kernel option must reach the same fixed point (bit-exact depths)."""
    g = inputs.rmat(15, 16, 2, symmetric=True)
    rp, col = g.numpy()
    for s in inputs.bfs_sources(g, 2, seed=5):
        run_and_check(rp, col, s, **opts)
    gg = inputs.road_grid(80, 60, seed=3)
    rp, col = gg.numpy()
    run_and_check(rp, col, 0, **opts)


def test_virtual_ranks_tiny_packets_and_grid_bands():
    g = inputs.road_grid(120, 100, seed=1)
    rp, col = g.numpy()
    run_and_check(rp, col, 0, virtual_ranks=4, agg_batch_msgs=1, channel_packets=2)
    run_and_check(rp, col, 777, virtual_ranks=8, agg_batch_msgs=7, agg_max_age_ns=0, channel_packets=4)


def test_bad_arguments():
    rp, col = csr_of(3, [(0, 1)])
    with atos.Graph(rp, col) as G:
        for bad in (-1, 3):
            with pytest.raises(atos.AtosError) as e:
                G.bfs(bad)
            assert e.value.status == 1
    with pytest.raises(atos.AtosError):
        atos.Graph(rp, np.array([7], dtype=np.int32))          # col out of range
    with pytest.raises(atos.AtosError):
        atos.Graph(rp, col, device=64)


@pytest.mark.slow
@pytest.mark.parametrize("vr", [2, 4, 8])
def test_rmat24_config2_full_size_virtual_ranks(vr):
    """configs[2] at full size with the multi-rank protocol (2/4/8 ranks, virtual on
    this one GPU): depths and min-id parents bit-exact vs the oracle, aggregation
    on and off (identical depth arrays for p in {1,2,4,8})."""
    g = inputs.make_config("rmat24", device="cuda")
    src = inputs.bfs_sources(g, 3)[vr.bit_length() - 2]
    rpn, coln = g.numpy()
    want = oracle.bfs(rpn, coln, src)
    pwant = oracle.bfs_parents_minid(rpn, coln, want, src)
    for agg in (1, 0):
        with atos.Graph(g.row_ptr, g.col, g.n, virtual_ranks=vr, agg_enabled=agg) as G:
            d, par = G.bfs(src, parent=True)
        assert np.array_equal(d, want), (vr, agg)
        assert np.array_equal(par, pwant), (vr, agg)


@pytest.mark.slow
@pytest.mark.parametrize("pq", [-1, 0])
def test_rmat24_config2_full_size(pq):
    """BASELINE configs[2] at full size: the launch configuration bench.py times
    (auto: level buckets) and the FIFO queue with the byte filter."""
    g = inputs.make_config("rmat24", device="cuda")
    rp, col = g.row_ptr, g.col
    srcs = inputs.bfs_sources(g, 2)
    rpn, coln = g.numpy()
    with atos.Graph(rp, col, pq_delta=pq) as G:
        for s in srcs:
            d = G.bfs(s)
            want = oracle.bfs(rpn, coln, s)
            assert np.array_equal(d, want)


@pytest.mark.parametrize("opts", [dict(relabel=0), dict(relabel=1, hub_cache=0), dict(relabel=1),
                                  dict(relabel=0, hub_cache=1024), dict(relabel=1, relax_red=0),
                                  dict(relabel=1, probe_filter=1), dict(relabel=1, pipeline=1),
                                  dict(relabel=1, pipeline=0, hub_cache=128),
                                  dict(relabel=1, hub_cache=128 * 3), dict(relabel=1, hub_cache=1 << 22),
                                  dict(relabel=1, virtual_ranks=4, hub_cache=128),
                                  dict(relabel=1, virtual_ranks=3, hub_cache=96 * 64),
                                  dict(relabel=1, virtual_ranks=8, agg_enabled=0)])
def test_relabel_and_hub_cache_same_depths_and_parents(opts):
    """Degree relabeling and the hub bounds (atos_bfs1.cuh: per-128-hub chunk
    upper bounds in shared memory) change the internal order and retire edges
    without a probe; depths and the min-id parents in the caller's ids must be
    unchanged."""
    g = inputs.rmat(15, 16, 4, symmetric=True)
    rp, col = g.numpy()
    for s in inputs.bfs_sources(g, 2, seed=7):
        run_and_check(rp, col, s, **opts)
    gg = inputs.road_grid(70, 50, seed=4)
    rp, col = gg.numpy()
    run_and_check(rp, col, 3, **opts)
    rng = np.random.default_rng(11)
    n = 1500
    edges = list(zip(rng.integers(0, n, 5000).tolist(), (rng.integers(0, n, 5000) // 7).tolist()))
    rp, col = csr_of(n, edges)        # skewed in-degree, dangling rows, duplicates
    run_and_check(rp, col, int(edges[0][0]), **opts)


def test_hub_cache_active_on_skewed_graph():
    """On a skewed graph most edges point at hubs whose chunk bound is already
    small: the hub bounds retire a large share of the edges without a probe."""
    g = inputs.rmat(18, 16, 1, symmetric=True)
    rp, col = g.numpy()
    src = inputs.bfs_sources(g, 1)[0]
    with atos.Graph(rp, col, relabel=1, hub_cache=65536) as G:
        d, st = G.bfs(src, stats=True)
    assert np.array_equal(d, oracle.bfs(rp, col, src))
    assert st["hub_hits"] > 0.2 * st["edges"], st
    with atos.Graph(rp, col, hub_cache=0) as G:
        d, st = G.bfs(src, stats=True)
    assert np.array_equal(d, oracle.bfs(rp, col, src)) and st["hub_hits"] == 0


@pytest.mark.parametrize("opts", [dict(split_edges=256), dict(split_edges=256, relabel=0),
                                  dict(split_edges=256, virtual_ranks=4), dict(split_edges=256, virtual_ranks=3,
                                                                               agg_enabled=0),
                                  dict(split_edges=512, keep_items=64, fetch_size=5),
                                  dict(split_edges=256, probe_filter=1), dict(split_edges=0)])
def test_row_splitting_same_depths_and_parents(opts):
    """Hub rows cut into pieces any worker can pop
    must reach the same depths and min-id parents."""
    g = inputs.rmat(15, 16, 3, symmetric=True)
    rp, col = g.numpy()
    for s in inputs.bfs_sources(g, 2, seed=9):
        run_and_check(rp, col, s, **opts)
    # a star + path: hub 0 of degree 60000 feeding a chain, and a second hub beyond id 65535
    n = 140000
    edges = [(0, v) for v in range(1, 60001)] + [(v, 0) for v in range(1, 60001)]
    edges += [(v, v + 1) for v in range(60000, 70000)] + [(v + 1, v) for v in range(60000, 70000)]
    edges += [(70000, v) for v in range(70001, n)] + [(v, 70000) for v in range(70001, n)]
    rp, col = csr_of(n, edges)
    for s in (0, 5, 70000, 139999):
        run_and_check(rp, col, s, **opts)


def test_row_splitting_publishes_pieces():
    n = 50001
    edges = [(0, v) for v in range(1, n)] + [(v, 0) for v in range(1, n)]
    rp, col = csr_of(n, edges)
    with atos.Graph(rp, col, split_edges=256) as G:
        d, st = G.bfs(0, stats=True)
    assert np.array_equal(d, oracle.bfs(rp, col, 0))
    # the hub's row (50000 edges) becomes 1 kept + 195 published pieces
    assert st["pops"] >= n + 195, st
    assert st["edges"] == col.size, st


@pytest.mark.parametrize("opts", [dict(discrete=1), dict(discrete=1, split_edges=256), dict(discrete=1, keep_items=0),
                                  dict(discrete=1, keep_items=64, keep_mode=1), dict(discrete=1, probe_filter=1)])
def test_discrete_kernel_mode_same_depths_and_parents(opts):
    """one worker launch per queue snapshot, looped by a CUDA-graph
    while-node, reaches the same depths and min-id parents."""
    g = inputs.rmat(15, 16, 6, symmetric=True)
    rp, col = g.numpy()
    for s in inputs.bfs_sources(g, 2, seed=3):
        run_and_check(rp, col, s, **opts)
    gg = inputs.road_grid(60, 40, seed=2)
    rp, col = gg.numpy()
    run_and_check(rp, col, 5, **opts)


def test_discrete_iterations_equal_levels_on_a_path():
    n = 1000
    rp, col = csr_of(n, [(i, i + 1) for i in range(n - 1)] + [(i + 1, i) for i in range(n - 1)])
    with atos.Graph(rp, col, discrete=1, keep_items=0) as G:
        d, st = G.bfs(0, stats=True)
        assert np.array_equal(d, np.arange(n))
        assert st["iterations"] == n, st
        d2, st2 = G.bfs(n - 1, stats=True)            # repeated solve on the same instantiated graph
        assert np.array_equal(d2, np.arange(n)[::-1]) and st2["iterations"] == n
    with pytest.raises(atos.AtosError):
        atos.Graph(rp, col, discrete=1, virtual_ranks=2)


@pytest.mark.parametrize("chunk", ["7", "1000", "100003"])
def test_streamed_relabel_load_from_host(chunk, monkeypatch):
    """Host CSR + relabeling streams the columns through the permutation in chunks
    (graph_load); chunk boundaries inside rows must not change anything."""
    monkeypatch.setenv("ATOS_LOAD_CHUNK", chunk)
    g = inputs.rmat(14, 16, 8, symmetric=True)
    rp, col = g.numpy()
    for s in inputs.bfs_sources(g, 2, seed=4):
        run_and_check(rp, col, s, relabel=1)
    bad = col.copy()
    bad[len(bad) // 2] = g.n + 5                        # out-of-range column id inside a late chunk
    with pytest.raises(atos.AtosError) as e:
        atos.Graph(rp, bad, relabel=1)
    assert e.value.status == 1


@pytest.mark.parametrize("chunk", ["100003", "30000"])
def test_streamed_relabel_long_rows(chunk, monkeypatch):
    """Rows with more than 8192 edges inside one load chunk go to the one-CTA-per-row
    permutation kernel (graph_load's streamed relabeling)."""
    monkeypatch.setenv("ATOS_LOAD_CHUNK", chunk)
    n = 40000
    hub = torch.zeros(n - 1, dtype=torch.int64)
    leaves = torch.arange(1, n, dtype=torch.int64)
    chain = torch.arange(1, n - 1, dtype=torch.int64)
    src_e = torch.cat([hub, chain, torch.full((n - 2,), 7, dtype=torch.int64)])
    dst_e = torch.cat([leaves, chain + 1, torch.arange(2, n, dtype=torch.int64)])
    keep = src_e != dst_e
    rp, col = inputs.csr_from_edges(n, src_e[keep], dst_e[keep], symmetrize=True).numpy()
    assert np.diff(rp).max() > 3 * 8192
    for s in (0, 123, n - 1):
        run_and_check(rp, col, s, relabel=1)


def bfs_properties_hold(rp_dev, col_dev, depth_dev, src):
    """Properties that fix BFS depths on a symmetric graph at any size (checked on
    the GPU with plain torch ops): depth(src) = 0; |d(u) - d(v)| <= 1 on every edge
    between reached vertices; no edge from a reached to an unreached vertex; every
    reached v != src has a neighbour at depth d(v) - 1."""
    n = rp_dev.numel() - 1
    deg = rp_dev[1:] - rp_dev[:-1]
    d = depth_dev.to(torch.int64)
    assert int(d[src]) == 0
    ok_all = True
    # process the edge list in slices to bound memory
    row = torch.repeat_interleave(torch.arange(n, device=d.device), deg)
    has_parent = torch.zeros(n, dtype=torch.bool, device=d.device)
    step = 1 << 28
    for a in range(0, col_dev.numel(), step):
        u = row[a:a + step]
        v = col_dev[a:a + step].to(torch.int64)
        du, dv = d[u], d[v]
        ru, rv = du >= 0, dv >= 0
        ok_all &= bool(((ru & rv) <= ((du - dv).abs() <= 1)).all())
        ok_all &= bool((ru <= rv).all())
        par = ru & rv & (du == dv - 1)
        has_parent[v[par]] = True
    reached = d >= 0
    reached[src] = False
    ok_all &= bool((reached <= has_parent).all())
    return ok_all


@pytest.mark.slow
def test_rmat26_north_star_full_size():
    """The north-star graph (RMAT-26 ef16 symmetric, 2.1 G CSR entries) in the bench's
    launch configuration: bit-exact vs the oracle's serial BFS from one source, and
    the BFS properties on the GPU from a second."""
    g = inputs.make_config("rmat26", device="cuda")
    srcs = inputs.bfs_sources(g, 2)
    depth = torch.empty(g.n, dtype=torch.int32, device="cuda")
    with atos.Graph(g.row_ptr, g.col, g.n) as G:
        G.bfs(srcs[1], depth_out=depth)
        G.sync()
        assert bfs_properties_hold(g.row_ptr, g.col, depth, srcs[1])
        d0, st = G.bfs(srcs[0], stats=True)
    # the default (pq_delta = -1, auto) orders this graph by level buckets (N1)
    assert st["pq_buckets"] > 0
    rpn, coln = g.numpy()
    assert np.array_equal(d0, oracle.bfs(rpn, coln, srcs[0]))


@pytest.mark.slow
def test_grid4900_config3_full_size():
    """BASELINE configs[3] (road-like grid, 24 M vertices, ~11.8 K levels) at full size,
    from the corner (the bench source) and the centre."""
    g = inputs.make_config("grid4900", device="cuda")
    rpn, coln = g.numpy()
    with atos.Graph(g.row_ptr, g.col, g.n) as G:
        for s in (0, g.n // 2 + 2450):
            assert np.array_equal(G.bfs(s), oracle.bfs(rpn, coln, s))


@pytest.mark.parametrize("opts", [dict(), dict(split_edges=0), dict(split_edges=256), dict(hub_cache=0),
                                  dict(fetch_size=3), dict(keep_items=64, keep_mode=1)])
def test_bfs1_long_rows_alignment_and_chunk_map(opts):
    """The single-rank expansion (atos_bfs1.cuh): rows of >= 128 edges start at every
    alignment mod 4 and end ragged; a row of 700 000 edges without splitting has more
    128-edge chunks than the per-batch chunk map (4096) and takes the search path;
    the last row of the column array is long (16-B loads past its end read the
    array's padding)."""
    rng = np.random.default_rng(5)
    n = 800000
    edges = [(0, v) for v in range(1, 700001)]                       # one huge row (unsplittable with split 0)
    for u in range(1, 3000):                                          # long rows of every length mod 4
        d = 128 + int(rng.integers(0, 400))
        edges += [(u, int(x)) for x in rng.integers(1, n, d)]
    edges += [(n - 1, int(x)) for x in rng.integers(0, n, 300)]       # long last row
    edges += [(v, 0) for v in range(1, 700001, 7)]                   # back edges to the hub
    rp, col = csr_of(n, list(set(edges)))
    for s in (0, 1, 17, n - 1):
        run_and_check(rp, col, s, **opts)

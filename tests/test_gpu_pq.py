"""GPU parity of the BFS priority queue (Listing 4's
DistributedPriorityQueues(threshold, threshold_delta); its
effect on redundant work, Table III).

The priority queue only reorders work, so depths must stay bit-exact and the
min-id parents equal to the oracle's.  One property is specific to it: with
threshold_delta = 1 on one rank, buckets are BFS levels, every vertex is
expanded exactly once at its final depth, so the edges scanned equal
m_reached exactly and the number of bucket advances equals the eccentricity
of the source.
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs

from test_gpu_bfs import check_parents

pytestmark = pytest.mark.gpu


def m_reached(rp, depth):
    deg = np.diff(rp)
    return int(deg[depth >= 0].sum())


def run_pq(rp, col, src, **cfg):
    with atos.Graph(rp, col, **cfg) as G:
        d, par, st = G.bfs(src, parent=True, stats=True)
    want = oracle.bfs(rp, col, src)
    assert np.array_equal(d, want), f"first diff at {np.nonzero(d != want)[0][:5]}"
    check_parents(rp, col, d, par, src)
    assert np.array_equal(par, oracle.bfs_parents_minid(rp, col, want, src))
    return d, st


@pytest.mark.parametrize("delta", [1, 2, 3, 64])
@pytest.mark.parametrize("graph", ["rmat14", "grid"])
def test_pq_same_depths_and_parents(graph, delta):
    g = inputs.rmat(14, 16, 1, symmetric=True) if graph == "rmat14" else inputs.road_grid(120, 90, 1)
    rp, col = g.numpy()
    src = inputs.bfs_sources(g, 1)[0] if graph == "rmat14" else 0
    d, st = run_pq(rp, col, src, pq_delta=delta)
    if delta < d.max():
        assert st["far_pushes"] > 0 and st["pq_buckets"] > 0


@pytest.mark.parametrize("graph", ["rmat14", "grid", "path"])
def test_pq_delta1_is_level_synchronous(graph):
    if graph == "path":
        n = 3000
        idx = np.arange(n - 1)
        rp, col = inputs.csr_from_edges(n, torch.from_numpy(idx), torch.from_numpy(idx + 1), symmetrize=True).numpy()
        src = 0
    else:
        g = inputs.rmat(14, 16, 2, symmetric=True) if graph == "rmat14" else inputs.road_grid(200, 150, 2)
        rp, col = g.numpy()
        src = inputs.bfs_sources(g, 1)[0] if graph == "rmat14" else 0
    for opts in (dict(), dict(split_edges=256), dict(keep_items=64, keep_mode=1)):   # keeping is off under pq
        d, st = run_pq(rp, col, src, pq_delta=1, **opts)
        assert st["edges"] == m_reached(rp, d), (opts, st["edges"], m_reached(rp, d))
        assert st["pq_buckets"] == d.max(), (opts, st["pq_buckets"], d.max())


def test_pq_threshold_and_repeated_solves():
    # several solves on one handle: the bucket counter persists across solves (the
    # current ring alternates), every solve starts again at `threshold`
    g = inputs.rmat(13, 16, 3, symmetric=True)
    rp, col = g.numpy()
    with atos.Graph(rp, col, pq_delta=2, pq_threshold=5) as G:
        for s in inputs.bfs_sources(g, 5):
            d, st = G.bfs(s, stats=True)
            want = oracle.bfs(rp, col, s)
            assert np.array_equal(d, want)
            # the first bucket holds depths < 5, later ones 2 levels each
            assert st["pq_buckets"] == (0 if d.max() < 5 else (d.max() - 5) // 2 + 1)


@pytest.mark.parametrize("vr", [2, 4, 8])
@pytest.mark.parametrize("delta", [1, 4])
def test_pq_virtual_ranks(vr, delta):
    g = inputs.rmat(15, 16, 1, symmetric=True)
    rp, col = g.numpy()
    for s in inputs.bfs_sources(g, 2):
        run_pq(rp, col, s, pq_delta=delta, virtual_ranks=vr)


@pytest.mark.parametrize("opts", [dict(agg_enabled=0), dict(channel_packets=2, agg_batch_msgs=1)])
def test_pq_virtual_ranks_tiny_channels(opts):
    g = inputs.road_grid(100, 80, 3)
    rp, col = g.numpy()
    part = [0, 2000, 4000, 6000, 8000]
    with atos.Graph(rp, col, part=part, virtual_ranks=4, pq_delta=1, **opts) as G:
        d = G.bfs(0)
    assert np.array_equal(d, oracle.bfs(rp, col, 0))


@pytest.mark.parametrize("delta", [1, 3])
def test_pq_discrete_kernel_mode(delta):
    # the paper's fastest scale-free configuration: priority queue + discrete kernels
    g = inputs.rmat(14, 16, 4, symmetric=True)
    rp, col = g.numpy()
    src = inputs.bfs_sources(g, 1)[0]
    d, st = run_pq(rp, col, src, pq_delta=delta, discrete=1)
    if delta == 1:
        assert st["edges"] == m_reached(rp, d)
        assert st["pq_buckets"] == d.max()


def test_pq_pagerank_unaffected():
    g = inputs.rmat(12, 16, 1, symmetric=False)
    rp, col = g.numpy()
    with atos.Graph(rp, col, pq_delta=1) as G:
        rank, res = G.pagerank(0.85, 1e-9)
    p, _, _ = oracle.pagerank(rp, col, 0.85, 1e-12)
    p_hat = rank / rank.sum()
    assert np.abs(p_hat - p).max() <= 1e-6 and np.abs(p_hat - p).sum() <= 1e-5
    assert np.all(res < 1e-9)


def test_pq_rmat24_config2_full_size():
    g = inputs.make_config("rmat24", device="cuda")
    rp, col = g.numpy()
    src = inputs.bfs_sources(g, 1)[0]
    with atos.Graph(g.row_ptr, g.col, g.n, pq_delta=1) as G:
        d, st = G.bfs(src, stats=True)
    want = oracle.bfs(rp, col, src)
    assert np.array_equal(d, want)
    assert st["edges"] == m_reached(rp, d)


@pytest.mark.parametrize("var", ["ATOS_VIS_NOCLAIM", "ATOS_NO_VIS", "ATOS_NO_PQ_EARLY"])
def test_pq_delta1_switches(monkeypatch, var):
    # the level-bucket variants behind the A/B switches: discoverer
    # atomicOr instead of claim at pop; depth words + filter instead of the bitmap
    monkeypatch.setenv(var, "1")
    for g, src in ((inputs.rmat(15, 16, 2, symmetric=True), None), (inputs.road_grid(80, 60, 3), 0)):
        rp, col = g.numpy()
        s = inputs.bfs_sources(g, 1, seed=5)[0] if src is None else src
        d, st = run_pq(rp, col, s, pq_delta=1)
        assert st["pq_buckets"] == d.max()


def test_pq_auto_is_fifo_on_small_graphs():
    # auto (the default) keeps the FIFO queue below 2^20 vertices and on non-skewed graphs
    g = inputs.rmat(14, 16, 1, symmetric=True)
    rp, col = g.numpy()
    src = inputs.bfs_sources(g, 1)[0]
    with atos.Graph(rp, col) as G:
        d, st = G.bfs(src, stats=True)
    assert np.array_equal(d, oracle.bfs(rp, col, src))
    assert st["pq_buckets"] == 0 and st["far_pushes"] == 0

"""Pins for the CPU oracle (oracle/) against things other than itself.

BFS: exhaustive brute force over all 4-vertex digraphs (walk counting with
integer matrix powers), hand-worked fixture, closed forms, scipy csgraph,
invariants on a Kronecker instance.
PageRank: closed forms (cycle, star fixture, K_n, alpha=0, all-dangling,
single vertex), dense linear solve of the defining equations, networkx.
"""
import itertools
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import shortest_path

import oracle
from paper_conf_sc_chenbpbyo22_b200 import inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def csr_of(n, edges):
    edges = sorted(edges)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    for u, _ in edges:
        row_ptr[u + 1] += 1
    row_ptr = np.cumsum(row_ptr)
    col = np.array([v for _, v in edges], dtype=np.int32)
    return row_ptr, col


def csr_of_adj(adj):
    row_ptr = np.zeros(len(adj) + 1, dtype=np.int64)
    row_ptr[1:] = np.cumsum([len(a) for a in adj])
    col = np.array([v for a in adj for v in a], dtype=np.int32)
    return row_ptr, col


# ----------------------------------------------------------------------------- BFS
def brute_depth_matrix_powers(A, src):
    """depth(v) = smallest k with (A^k)[src, v] > 0 (walk counting), else -1."""
    n = A.shape[0]
    depth = np.full(n, -1)
    M = np.eye(n, dtype=np.int64)
    for k in range(n):
        reach = M[src] > 0
        newly = reach & (depth < 0)
        depth[newly] = k
        M = np.minimum(M @ A, 1)           # clamp: only positivity matters
    return depth


def test_bfs_exhaustive_all_4_vertex_digraphs():
    n = 4
    pairs = [(u, v) for u in range(n) for v in range(n) if u != v]
    assert len(pairs) == 12
    for mask in range(1 << 12):
        edges = [pairs[i] for i in range(12) if mask >> i & 1]
        rp, col = csr_of(n, edges)
        A = np.zeros((n, n), dtype=np.int64)
        for u, v in edges:
            A[u, v] = 1
        for src in range(n):
            got = oracle.bfs(rp, col, src)
            want = brute_depth_matrix_powers(A, src)
            assert np.array_equal(got, want), (edges, src, got, want)


def test_bfs_hand_fixture():
    fx = json.load(open(os.path.join(GOLDEN, "bfs_hand.json")))
    rp, col = csr_of_adj(fx["adj"])
    assert oracle.bfs(rp, col, fx["src"]).tolist() == fx["depth"]


@pytest.mark.parametrize("n", [1, 2, 7, 50])
def test_bfs_closed_forms(n):
    # directed path 0->1->...->n-1: d(i) = i ; from the end only itself
    rp, col = csr_of(n, [(i, i + 1) for i in range(n - 1)])
    assert oracle.bfs(rp, col, 0).tolist() == list(range(n))
    assert oracle.bfs(rp, col, n - 1).tolist() == [-1] * (n - 1) + [0]
    # undirected cycle: d(i) = min(i, n-i)
    if n >= 3:
        e = [(i, (i + 1) % n) for i in range(n)] + [((i + 1) % n, i) for i in range(n)]
        rp, col = csr_of(n, e)
        assert oracle.bfs(rp, col, 0).tolist() == [min(i, n - i) for i in range(n)]
    # complete digraph: all 1
    e = [(u, v) for u in range(n) for v in range(n) if u != v]
    rp, col = csr_of(n, e)
    assert oracle.bfs(rp, col, 0).tolist() == [0] + [1] * (n - 1)
    # undirected star centre 0: from centre 1, from a leaf 1 (centre) / 2 (other leaves)
    if n >= 3:
        e = [(0, i) for i in range(1, n)] + [(i, 0) for i in range(1, n)]
        rp, col = csr_of(n, e)
        assert oracle.bfs(rp, col, 0).tolist() == [0] + [1] * (n - 1)
        want = [1] + [2] * (n - 1)
        want[1] = 0
        assert oracle.bfs(rp, col, 1).tolist() == want


def test_bfs_disconnected_and_isolated_source():
    rp, col = csr_of(6, [(0, 1), (1, 0), (2, 3), (3, 4)])
    assert oracle.bfs(rp, col, 0).tolist() == [0, 1, -1, -1, -1, -1]
    assert oracle.bfs(rp, col, 5).tolist() == [-1] * 5 + [0]
    assert oracle.bfs(rp, col, 2).tolist() == [-1, -1, 0, 1, 2, -1]


def test_bfs_bad_args():
    rp, col = csr_of(3, [(0, 1)])
    with pytest.raises(ValueError):
        oracle.bfs(rp, col, 3)
    with pytest.raises(ValueError):
        oracle.bfs(rp, col, -1)


def _scipy_depth(rp, col, src):
    n = rp.size - 1
    A = sp.csr_matrix((np.ones(col.size), col.astype(np.int64), rp), shape=(n, n))
    d = shortest_path(A, directed=True, unweighted=True, indices=src)
    return np.where(np.isinf(d), -1, d).astype(np.int64)


@pytest.mark.parametrize("seed", range(12))
def test_bfs_random_vs_scipy(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 65))
    m = int(rng.integers(0, 4 * n))
    # multi-edges and self-loops allowed: multiplicity must not matter for depths
    edges = list(zip(rng.integers(0, n, m).tolist(), rng.integers(0, n, m).tolist()))
    rp, col = csr_of(n, edges)
    for src in rng.integers(0, n, 3).tolist():
        assert np.array_equal(oracle.bfs(rp, col, src), _scipy_depth(rp, col, src))


def check_bfs_invariants(rp, col, src, d):
    n = rp.size - 1
    src_of = np.repeat(np.arange(n), np.diff(rp))
    assert d[src] == 0
    du, dv = d[src_of], d[col]
    reached_u = du >= 0
    # a reached vertex never has an unreached out-neighbour, and d(v) <= d(u)+1 on edges
    assert np.all(dv[reached_u] >= 0)
    assert np.all(dv[reached_u] <= du[reached_u] + 1)
    # every reached v != src has an in-neighbour at depth d(v)-1
    ok = np.zeros(n, dtype=bool)
    good = reached_u & (dv == du + 1)
    ok[col[good]] = True
    ok[src] = True
    assert np.all(ok[d >= 0])


def test_bfs_kron12_vs_scipy_and_invariants():
    g = inputs.make_config("kron12")
    rp, col = g.numpy()
    d = oracle.bfs(rp, col, 0)
    assert np.array_equal(d, _scipy_depth(rp, col, 0))
    check_bfs_invariants(rp, col, 0, d)
    # symmetric graph: |d(u) - d(v)| <= 1 on every edge with both ends reached
    src_of = np.repeat(np.arange(g.n), np.diff(rp))
    both = (d[src_of] >= 0) & (d[col] >= 0)
    assert np.all(np.abs(d[src_of][both] - d[col][both]) <= 1)
    assert (d >= 0).sum() > 3000 and d.max() <= 4


def test_parents_minid_by_rule():
    rng = np.random.default_rng(5)
    for _ in range(10):
        n = int(rng.integers(2, 40))
        m = int(rng.integers(0, 5 * n))
        edges = list(zip(rng.integers(0, n, m).tolist(), rng.integers(0, n, m).tolist()))
        rp, col = csr_of(n, edges)
        src = int(rng.integers(0, n))
        d = oracle.bfs(rp, col, src)
        par = oracle.bfs_parents_minid(rp, col, d, src)
        eset = set(edges)
        for v in range(n):
            if d[v] < 0:
                assert par[v] == -1
            elif v == src:
                assert par[v] == src
            else:
                cands = sorted(u for (u, w) in eset if w == v and d[u] == d[v] - 1)
                assert par[v] == cands[0]


# ----------------------------------------------------------------------------- PageRank
def dense_pagerank(n, edges, alpha):
    """Solve the defining linear system directly: (I - a M) p = (1-a)/n 1,
    M = P^T + (1/n) 1 d^T, with P[v,u] = mult(v->u)/outdeg(v), d = dangling indicator."""
    P = np.zeros((n, n))
    out = np.zeros(n)
    for u, v in edges:
        out[u] += 1
    for u, v in edges:
        P[u, v] += 1.0 / out[u]
    dang = (out == 0).astype(float)
    M = P.T + np.outer(np.ones(n), dang) / n
    p = np.linalg.solve(np.eye(n) - alpha * M, np.full(n, (1 - alpha) / n))
    return p / p.sum()


@pytest.mark.parametrize("n", [3, 10, 101])
def test_pr_cycle_is_uniform(n):
    rp, col = csr_of(n, [(i, (i + 1) % n) for i in range(n)])
    p, it, delta = oracle.pagerank(rp, col, 0.85)
    assert np.allclose(p, 1.0 / n, atol=1e-14, rtol=0)


def test_pr_star_golden():
    fx = json.load(open(os.path.join(GOLDEN, "star5_pagerank.json")))
    k = fx["k"]
    e = [(0, i) for i in range(1, k + 1)] + [(i, 0) for i in range(1, k + 1)]
    rp, col = csr_of(k + 1, e)
    p, _, _ = oracle.pagerank(rp, col, fx["alpha"])
    assert abs(p[0] - fx["p_center"]) < 1e-12
    assert np.all(np.abs(p[1:] - fx["p_leaf"]) < 1e-12)


@pytest.mark.parametrize("n", [1, 2, 5, 30])
def test_pr_symmetric_closed_forms(n):
    e = [(u, v) for u in range(n) for v in range(n) if u != v]
    rp, col = csr_of(n, e)
    p, _, _ = oracle.pagerank(rp, col, 0.85)
    assert np.allclose(p, 1.0 / n, atol=1e-14, rtol=0)           # K_n (and single vertex)
    rp, col = csr_of(n, [])
    p, _, _ = oracle.pagerank(rp, col, 0.85)
    assert np.allclose(p, 1.0 / n, atol=1e-14, rtol=0)           # all dangling


def test_pr_alpha_zero_uniform():
    rng = np.random.default_rng(3)
    edges = list(zip(rng.integers(0, 20, 60).tolist(), rng.integers(0, 20, 60).tolist()))
    rp, col = csr_of(20, edges)
    p, it, _ = oracle.pagerank(rp, col, 0.0)
    assert np.allclose(p, 1.0 / 20, atol=1e-15, rtol=0)


@pytest.mark.parametrize("seed", range(10))
def test_pr_vs_dense_solve(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(2, 120))
    m = int(rng.integers(0, 6 * n))
    # dangling vertices, self-loops and multi-edges all present
    edges = list(zip(rng.integers(0, n, m).tolist(), rng.integers(0, n, m).tolist()))
    rp, col = csr_of(n, edges)
    alpha = float(rng.choice([0.5, 0.85, 0.95]))
    p, it, delta = oracle.pagerank(rp, col, alpha, tol=1e-14)
    want = dense_pagerank(n, edges, alpha)
    assert abs(p.sum() - 1.0) < 1e-12
    assert np.max(np.abs(p - want)) < 1e-11, (n, alpha)


def test_pr_kron10_vs_networkx():
    nx = pytest.importorskip("networkx")
    g = inputs.rmat(10, 16, 2, symmetric=False, permute=True)
    rp, col = g.numpy()
    p, it, delta = oracle.pagerank(rp, col, 0.85, tol=1e-13)
    G = nx.DiGraph()
    G.add_nodes_from(range(g.n))
    src_of = np.repeat(np.arange(g.n), np.diff(rp))
    G.add_edges_from(zip(src_of.tolist(), col.tolist()))
    ref = nx.pagerank(G, alpha=0.85, tol=1e-15, max_iter=10000)
    ref = np.array([ref[i] for i in range(g.n)])
    assert np.abs(p - ref).sum() < 1e-10
    assert (np.diff(rp) == 0).sum() > 0              # dangling vertices exercised


def test_pr_thread_count_invariant():
    g = inputs.rmat(12, 16, 1, symmetric=False)
    rp, col = g.numpy()
    p1, it1, _ = oracle.pagerank(rp, col, 0.85, nthreads=1)
    p4, it4, _ = oracle.pagerank(rp, col, 0.85, nthreads=4)
    assert it1 == it4 and np.array_equal(p1, p4)


def test_pr_not_converged_is_an_error():
    """The oracle's answer is the fixed point to ||dp||_1 <= tol (north_star: Jacobi
    iterated to a 1e-12 L1 residual); a run cut off by max_iter must not silently
    become an expected value."""
    g = inputs.rmat(10, 16, 3, symmetric=False)
    rp, col = g.numpy()
    with pytest.raises(RuntimeError, match="did not converge"):
        oracle.pagerank(rp, col, 0.85, tol=1e-12, max_iter=3)
    p, it, delta = oracle.pagerank(rp, col, 0.85, tol=1e-12)
    assert delta <= 1e-12 and it > 3

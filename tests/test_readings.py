"""Checks of DESIGN.md's readings of the paper's under-specified PageRank.

PAPER.md:1168-1182 (Sec. IV 'PageRank') gives the push-residual method in prose
only.  DESIGN.md readings R2-R6 fix: rank=0, residual=1-alpha, every vertex
enqueued; pop v -> rank += r, push alpha*r/outdeg to out-neighbours; dangling
vertices absorb; eps is an absolute bound on the unnormalised residual;
re-enqueue on the crossing old < eps <= old+delta.

Here a serial pure-Python model of exactly that rule (a model of the GPU
method, independent of both the CUDA path and the oracle) is checked against
the oracle's PageRank within the bound the readings imply:
||p_hat - p||_1 <= 2 eps / (1-alpha)^2, and the queue-empty state implies
every residual < eps.
"""
from collections import deque

import numpy as np
import pytest

import oracle
from paper_conf_sc_chenbpbyo22_b200 import inputs


def push_pagerank_model(rp, col, alpha, eps):
    n = rp.size - 1
    rank = np.zeros(n)
    res = np.full(n, 1.0 - alpha)
    q = deque(range(n))
    pops = 0
    while q:
        v = q.popleft()
        pops += 1
        r = res[v]
        res[v] = 0.0
        rank[v] += r
        deg = rp[v + 1] - rp[v]
        if deg == 0:
            continue                        # dangling: absorb (reading R4)
        d = alpha * r / deg
        for e in range(rp[v], rp[v + 1]):
            u = col[e]
            old = res[u]
            res[u] = old + d
            if old < eps <= old + d:        # crossing enqueue (reading R5)
                q.append(u)
    return rank, res, pops


@pytest.mark.parametrize("seed,alpha", [(1, 0.85), (2, 0.85), (3, 0.5)])
def test_push_model_reaches_oracle_within_bound(seed, alpha):
    g = inputs.rmat(8, 8, seed, symmetric=False)
    rp, col = g.numpy()
    eps = 1e-7
    rank, res, pops = push_pagerank_model(rp, col, alpha, eps)
    assert np.all(res < eps) and np.all(res >= 0)
    p_hat = rank / rank.sum()
    p, _, _ = oracle.pagerank(rp, col, alpha, tol=1e-14)
    bound = 2 * eps / (1 - alpha) ** 2
    assert np.abs(p_hat - p).sum() <= bound
    # invariant of the push method: rank + (I - a P^T)^-1 res == (1-a)(I - a P^T)^-1 1
    n = g.n
    P = np.zeros((n, n))
    deg = np.diff(rp)
    src = np.repeat(np.arange(n), deg)
    np.add.at(P, (src, col), 1.0 / deg[src])
    Minv = np.linalg.inv(np.eye(n) - alpha * P.T)
    assert np.allclose(rank + Minv @ res, (1 - alpha) * Minv @ np.ones(n), atol=1e-10)

"""The worker's queue: PAPER.md Fig. 1's push / pop /
push-then-pop microbenchmark run by libatos on the
worker's own ring code (atos_queue_bench), checked for multiset conservation --
no item lost or duplicated -- under thread / warp / CTA workers, FETCH_SIZE
below the worker size, CAS reservation, tiny rings that wrap many laps, and
queue indices that cross 2^32 (the slots carry 32-bit tags of u64 indices;
Listing 6's counter is a 32-bit reserv_index).  The solver itself is
also run with every ring index starting just below 2^32."""
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NEAR_2_32 = (1 << 32) - 3000


def pushed_items(threads, rounds):
    return np.arange(threads * rounds, dtype=np.uint32)


@pytest.mark.parametrize("worker,fetch", [(1, 1), (32, 32), (32, 8), (512, 512), (512, 64), (512, 1)])
@pytest.mark.parametrize("op", ["push_then_pop", "pop"])
def test_queue_conservation(worker, fetch, op):
    threads, rounds = 1 << 14, 10
    ms, popped = atos.queue_bench(worker, op, threads, rounds, fetch_size=fetch, popped=True)
    assert ms > 0
    assert np.array_equal(np.sort(popped), pushed_items(threads, rounds))


@pytest.mark.parametrize("worker", [1, 32, 512])
def test_queue_cas_reservation(worker):
    threads, rounds = 4096, 10
    _, popped = atos.queue_bench(worker, "push_then_pop", threads, rounds, reserve_cas=True, popped=True)
    assert np.array_equal(np.sort(popped), pushed_items(threads, rounds))


@pytest.mark.parametrize("worker", [32, 512])
def test_queue_tiny_ring_wraps_and_crosses_2_32(worker):
    # a ring of 2^13 slots for 40 * 2^13 push-then-pop pairs: 40 laps, and the u64
    # indices start just below 2^32, so every 32-bit slot tag wraps mid-run
    threads, rounds = 1 << 13, 40
    _, popped = atos.queue_bench(worker, "push_then_pop", threads, rounds, ring_cap=threads,
                                 index_base=NEAR_2_32, popped=True)
    assert np.array_equal(np.sort(popped), pushed_items(threads, rounds))


def test_queue_push_only_fills_exactly():
    threads, rounds = 1 << 12, 16
    ms, _ = atos.queue_bench(32, "push", threads, rounds, ring_cap=threads * rounds, index_base=NEAR_2_32)
    assert ms > 0


def _run_child(code, env_extra):
    env = dict(os.environ, **env_extra)
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    return r.stdout


def test_solver_ring_indices_cross_2_32():
    # ATOS_TEST_RING_BASE (test-only, read at graph_load): every ring of the handle
    # starts at index 2^32 - 3000; several PageRank solves push ~30 entries per
    # vertex, BFS solves (FIFO and priority queue, 1 and 4 ranks) follow on the
    # same handles, all past the wrap of the 32-bit slot tags
    code = r'''
import numpy as np, oracle
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs
g = inputs.rmat(12, 16, 1, symmetric=True); rp, col = g.numpy()
gd = inputs.rmat(12, 16, 2, symmetric=False); rpd, cold = gd.numpy()
p, _, _ = oracle.pagerank(rpd, cold, 0.85, 1e-12)
for cfg in (dict(), dict(virtual_ranks=4), dict(pq_delta=1), dict(pq_delta=2, virtual_ranks=2)):
    with atos.Graph(rpd, cold, **cfg) as G:
        for _ in range(2):
            r, s = G.pagerank(0.85, 1e-9)
            ph = r / r.sum()
            assert np.abs(ph - p).max() <= 1e-6 and np.abs(ph - p).sum() <= 1e-5, cfg
    with atos.Graph(rp, col, **cfg) as G:
        for src in inputs.bfs_sources(g, 4):
            assert np.array_equal(G.bfs(src), oracle.bfs(rp, col, src)), cfg
print("ok")
'''
    assert "ok" in _run_child(code, {"ATOS_TEST_RING_BASE": str(NEAR_2_32)})

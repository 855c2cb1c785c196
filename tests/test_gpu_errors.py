"""T6 error paths: device errors are reported by the call that
retires the solve, outputs are declared invalid, and the handle recovers --
a single-process handle (one rank or virtual ranks) is reset to its
just-loaded state, so the next solve on it is correct again (checked against
the oracle).  Also: the runtime experiment switches reach the same fixed point,
and atos_graph_free returns the handle's memory to the device."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("vr", [1, 4])
@pytest.mark.parametrize("fault,status", [("capacity", 4), ("timeout", 5)])
def test_injected_device_error_then_recovery(monkeypatch, vr, fault, status):
    g = inputs.rmat(14, 16, 2, symmetric=True)
    rp, col = g.numpy()
    src = inputs.bfs_sources(g, 1)[0]
    want = oracle.bfs(rp, col, src)
    with atos.Graph(rp, col, virtual_ranks=vr) as G:
        monkeypatch.setenv("ATOS_TEST_FAULT", fault)
        with pytest.raises(atos.AtosError) as e:
            G.bfs(src)
        assert e.value.status == status
        monkeypatch.delenv("ATOS_TEST_FAULT")
        for _ in range(2):                       # the reset handle solves correctly, repeatedly
            assert np.array_equal(G.bfs(src), want)
        # and PageRank on the same handle after the BFS error
        rank, res = G.pagerank(0.85, 1e-9)
        assert np.all(res < 1e-9)


def test_real_watchdog_fires_on_a_busy_solve_and_handle_recovers():
    """watchdog_ms=1 on a PageRank that runs for several ms: the watchdog is checked
    on every worker iteration (busy or idle), so it fires; atos_set_watchdog then
    lifts it and the same handle converges to the oracle's PageRank."""
    g = inputs.rmat(17, 16, 1, symmetric=False)
    rp, col = g.numpy()
    with atos.Graph(rp, col, watchdog_ms=1) as G:
        with pytest.raises(atos.AtosError) as e:
            G.pagerank(0.85, 1e-12)
        assert e.value.status == 5
        G.set_watchdog(60000)
        rank, res = G.pagerank(0.85, 1e-9)
    p, _, _ = oracle.pagerank(rp, col, 0.85, 1e-12)
    err = np.abs(rank / rank.sum() - p)
    assert err.max() <= 1e-6 and err.sum() <= 1e-5 and np.all(res < 1e-9)


@pytest.mark.parametrize("var", ["ATOS_DYNAMIC_CHUNKS", "ATOS_NO_EDGE_MAP", "ATOS_EARLY", "ATOS_WARP_FLUSH"])
def test_runtime_switches_same_depths(monkeypatch, var):
    """Experiment switches read per solve select non-default code;
    every one must reach the oracle's depths and min-id parents."""
    monkeypatch.setenv(var, "1")
    for g, srcs in ((inputs.rmat(15, 16, 2, symmetric=True), None), (inputs.road_grid(80, 60, seed=3), [0])):
        rp, col = g.numpy()
        for s in (srcs or inputs.bfs_sources(g, 2, seed=5)):
            with atos.Graph(rp, col) as G:
                d, par = G.bfs(s, parent=True)
            want = oracle.bfs(rp, col, s)
            assert np.array_equal(d, want)
            assert np.array_equal(par, oracle.bfs_parents_minid(rp, col, want, s))


def test_free_returns_memory_to_the_device():
    """The library allocates from a private pool and trims it at free:
    a freed graph's memory is available to torch again."""
    g = inputs.rmat(20, 16, 1, symmetric=True, device="cuda")
    torch.cuda.synchronize()
    free0, _ = torch.cuda.mem_get_info()
    G = atos.Graph(g.row_ptr, g.col, g.n)
    free1, _ = torch.cuda.mem_get_info()
    assert free0 - free1 > g.nnz * 4          # at least the column copy is resident
    G.free()
    torch.cuda.synchronize()
    free2, _ = torch.cuda.mem_get_info()
    assert free0 - free2 < 64 << 20, (free0, free1, free2)


def test_retained_blocks_reused_then_released():
    """pool_retain = 1 parks a freed handle's large blocks for the next load of the same
    sizes (load/solve/free loops); results stay exact, and the next handle without
    pool_retain returns everything to the device at its free."""
    g = inputs.rmat(20, 16, 2, symmetric=True, device="cuda")
    rp, col = g.numpy()
    src = inputs.bfs_sources(g, 1)[0]
    want = oracle.bfs(rp, col, src)
    torch.cuda.synchronize()
    free0, _ = torch.cuda.mem_get_info()
    for _ in range(3):
        G = atos.Graph(rp, col, pool_retain=1)          # host CSR: streamed load, several >= 64 MB blocks
        assert np.array_equal(G.bfs(src), want)
        G.free()
    G = atos.Graph(g.row_ptr, g.col, g.n)
    assert np.array_equal(G.bfs(src), want)
    G.free()
    torch.cuda.synchronize()
    free1, _ = torch.cuda.mem_get_info()
    assert free0 - free1 < 64 << 20, (free0, free1)

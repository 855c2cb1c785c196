"""N>1 host-side logic on CPU (gloo, world_size 2): handle exchange in rank order,
peer connection through the Graph interface, max/sum over ranks, partition and
arena layout agreement across ranks."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class FakeGraph:
    """Stands in for atos.Graph: records what connect() receives."""

    def __init__(self, rank):
        self.rank = rank
        self.handles = None

    def export_handle(self):
        return bytes([self.rank]) * 64

    def connect(self, handles):
        self.handles = list(handles)


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    from paper_conf_sc_chenbpbyo22_b200 import atos
    from paper_conf_sc_chenbpbyo22_b200 import dist as adist
    r, w, _ = adist.init(backend="gloo")
    g = FakeGraph(r)
    adist.connect_graph(g, w)
    res = {
        "handles_ok": g.handles == [bytes([k]) * 64 for k in range(w)],
        "max": adist.max_over_ranks(float(r + 1)),
        "sum": adist.sum_over_ranks(float(r + 1)),
        "part": atos.partition_balanced(1000, w),
        "arena": atos.arena_bytes(1 << 14, w, r, channel_packets=16),
    }
    q.put((r, res))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_host_logic(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(world):
        assert out[r]["handles_ok"]
        assert out[r]["max"] == float(world)
        assert out[r]["sum"] == float(world * (world + 1) // 2)
        assert out[r]["part"] == out[0]["part"] == [(k * 1000) // world for k in range(world + 1)]
    assert all(out[r]["arena"] > (1 << 14) * 4 for r in range(world))

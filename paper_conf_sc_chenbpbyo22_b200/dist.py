"""Multi-process plumbing (one process per GPU, torch.distributed for setup only).

The peer mapping is the analogue of the paper's symmetric heap
(nvshmem_malloc, Listing 5): every rank exports one IPC handle of
its device arena; handles are all-gathered once through torch.distributed and
each rank maps every peer over NVLink.  Nothing here runs on the hot path.
"""
from __future__ import annotations

import os
from typing import Callable, List, Optional

import torch
import torch.distributed as dist


def env_rank_world():
    local = int(os.environ.get("LOCAL_RANK", os.environ.get("RANK", "0")))
    if os.environ.get("ATOS_SAME_DEVICE"):      # test mode: every rank on device 0 (time-sliced)
        local = 0
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), local


def init(backend: Optional[str] = None):
    """Initialise the default process group from torchrun env (127.0.0.1 rendezvous).
    Backend: ATOS_DIST_BACKEND, else NCCL with a GPU (gloo when ATOS_SAME_DEVICE is set,
    since NCCL refuses two ranks on one GPU), else gloo."""
    rank, world, local = env_rank_world()
    if world > 1 and not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        if backend is None:
            backend = os.environ.get("ATOS_DIST_BACKEND")
        if backend is None:
            backend = "nccl" if torch.cuda.is_available() and not os.environ.get("ATOS_SAME_DEVICE") else "gloo"
        if backend == "nccl":
            torch.cuda.set_device(local)
        dist.init_process_group(backend, rank=rank, world_size=world)
    return rank, world, local


def exchange_handles(my_handle: bytes, world: int) -> List[bytes]:
    """All-gather one fixed-size handle per rank, returned in rank order."""
    out: List[Optional[bytes]] = [None] * world
    dist.all_gather_object(out, my_handle)
    assert all(isinstance(h, (bytes, bytearray)) and len(h) == len(my_handle) for h in out)
    return [bytes(h) for h in out]


def connect_graph(graph, world: int):
    """graph: object with export_handle() and connect(handles) (atos.Graph)."""
    handles = exchange_handles(graph.export_handle(), world)
    graph.connect(handles)
    return handles


def load_distributed(row_ptr, col, n=None, part=None, graph_factory: Optional[Callable] = None, **cfg):
    """Load this rank's share of the graph and map every peer.  Collective."""
    rank, world, local = env_rank_world()
    if graph_factory is None:
        from . import atos
        graph_factory = atos.Graph
    g = graph_factory(row_ptr, col, n, part, rank=rank, n_ranks=world, device=local, **cfg)
    if world > 1:
        connect_graph(g, world)
        dist.barrier()
    return g


def max_over_ranks(x: float) -> float:
    """Max of a per-rank scalar (device time) across ranks; identity when single-process."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(x)
    dev = torch.device("cuda") if dist.get_backend() == "nccl" else torch.device("cpu")
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x: float) -> float:
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(x)
    dev = torch.device("cuda") if dist.get_backend() == "nccl" else torch.device("cpu")
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def max_over_ranks_vec(xs):
    """Element-wise max over ranks of a list of per-rank scalars (per-step device times)."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return [float(x) for x in xs]
    dev = torch.device("cuda") if dist.get_backend() == "nccl" else torch.device("cpu")
    t = torch.tensor([float(x) for x in xs], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return [float(v) for v in t.cpu().tolist()]

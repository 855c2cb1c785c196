"""Thin ctypes binding of the C ABI in include/atos.h (argument marshalling only).

Every step of the hot path runs in libatos.so's sm_100a kernels; this module
never computes anything itself and has no CPU fallback: if the library is
missing or CUDA is unavailable, calls fail loudly.

Names follow the C ABI: ``graph_load`` / ``bfs`` / ``pagerank`` /
``graph_free`` wrap ``atos_graph_load`` / ``atos_bfs`` / ``atos_pagerank`` /
``atos_graph_free``; ``Graph`` is the object form used by tests and bench.py.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence

import numpy as np

from . import _build

ATOS_MAX_RANKS = 8
ATOS_IPC_HANDLE_BYTES = 64

STATUS = {
    0: "ATOS_OK", 1: "ATOS_ERR_INVALID_ARG", 2: "ATOS_ERR_CUDA", 3: "ATOS_ERR_OOM",
    4: "ATOS_ERR_CAPACITY", 5: "ATOS_ERR_TIMEOUT", 6: "ATOS_ERR_PEER", 7: "ATOS_ERR_STATE",
}


class Config(ctypes.Structure):
    _fields_ = [
        ("worker_threads", ctypes.c_int32),
        ("ctas_per_sm", ctypes.c_int32),
        ("fetch_size", ctypes.c_int32),
        ("keep_items", ctypes.c_int32),
        ("l2_persist", ctypes.c_int32),
        ("prefetch", ctypes.c_int32),
        ("relax_red", ctypes.c_int32),
        ("pipeline", ctypes.c_int32),
        ("probe_filter", ctypes.c_int32),
        ("ring_cap_factor", ctypes.c_double),
        ("agg_enabled", ctypes.c_int32),
        ("agg_batch_msgs", ctypes.c_int32),
        ("agg_max_age_ns", ctypes.c_int64),
        ("channel_packets", ctypes.c_int32),
        ("watchdog_ms", ctypes.c_int64),
        ("rank", ctypes.c_int32),
        ("n_ranks", ctypes.c_int32),
        ("virtual_ranks", ctypes.c_int32),
        ("device", ctypes.c_int32),
        ("stream", ctypes.c_void_p),
        ("relabel", ctypes.c_int32),
        ("hub_cache", ctypes.c_int32),
        ("split_edges", ctypes.c_int32),
        ("keep_mode", ctypes.c_int32),
        ("discrete", ctypes.c_int32),
        ("pr_combine", ctypes.c_int32),
        ("pool_retain", ctypes.c_int32),
        ("pq_delta", ctypes.c_int32),
        ("pq_threshold", ctypes.c_int32),
    ]


class Stats(ctypes.Structure):
    _fields_ = [
        ("ms_worker", ctypes.c_double),
        ("ms_total", ctypes.c_double),
        ("pops", ctypes.c_uint64),
        ("edges", ctypes.c_uint64),
        ("local_pushes", ctypes.c_uint64),
        ("msgs_sent", ctypes.c_uint64),
        ("packets_sent", ctypes.c_uint64),
        ("bytes_sent", ctypes.c_uint64),
        ("idle_polls", ctypes.c_uint64),
        ("hub_hits", ctypes.c_uint64),
        ("busy_ns", ctypes.c_uint64),
        ("batches", ctypes.c_uint64),
        ("iterations", ctypes.c_uint64),
        ("far_pushes", ctypes.c_uint64),
        ("pq_buckets", ctypes.c_uint64),
        ("n_ranks", ctypes.c_int32),
        ("grid_ctas", ctypes.c_int32),
    ]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class QBenchConfig(ctypes.Structure):
    _fields_ = [
        ("worker_size", ctypes.c_int32),
        ("fetch_size", ctypes.c_int32),
        ("op", ctypes.c_int32),
        ("rounds", ctypes.c_int32),
        ("threads", ctypes.c_int64),
        ("ring_cap", ctypes.c_uint64),
        ("index_base", ctypes.c_uint64),
        ("reserve_cas", ctypes.c_int32),
        ("device", ctypes.c_int32),
    ]


class AtosError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


_lib = None

# (name, restype, argtypes) of every function declared in include/atos.h
_P = ctypes.c_void_p
_SIGS = [
    ("atos_config_init", ctypes.c_int, [ctypes.POINTER(Config)]),
    ("atos_partition_balanced", ctypes.c_int, [ctypes.c_int64, ctypes.c_int32, _P]),
    ("atos_validate_csr", ctypes.c_int, [_P, _P, ctypes.c_int64, ctypes.c_int64]),
    ("atos_arena_bytes", ctypes.c_int, [ctypes.c_int64, _P, ctypes.c_int32, ctypes.c_int32,
                                        ctypes.POINTER(Config), ctypes.POINTER(ctypes.c_uint64)]),
    ("atos_graph_load", ctypes.c_int, [_P, _P, ctypes.c_int64, ctypes.c_int64, _P,
                                       ctypes.POINTER(Config), ctypes.POINTER(_P)]),
    ("atos_graph_export", ctypes.c_int, [_P, _P]),
    ("atos_graph_connect", ctypes.c_int, [_P, _P]),
    ("atos_bfs", ctypes.c_int, [_P, ctypes.c_int64, _P, _P, ctypes.POINTER(Stats)]),
    ("atos_pagerank", ctypes.c_int, [_P, ctypes.c_double, ctypes.c_double, _P, _P, ctypes.POINTER(Stats)]),
    ("atos_set_watchdog", ctypes.c_int, [_P, ctypes.c_int64]),
    ("atos_sync", ctypes.c_int, [_P]),
    ("atos_last_stats", ctypes.c_int, [_P, ctypes.POINTER(Stats)]),
    ("atos_graph_free", ctypes.c_int, [_P]),
    ("atos_queue_bench", ctypes.c_int, [ctypes.POINTER(QBenchConfig), _P, ctypes.POINTER(ctypes.c_double)]),
    ("atos_last_error", ctypes.c_char_p, []),
    ("atos_version", ctypes.c_int32, []),
]
EXPORTED = [s[0] for s in _SIGS]


def lib_path() -> str:
    return _build.LIB


def load(build_if_missing: bool = True):
    """Load libatos.so (building it with nvcc if absent).  Raises if impossible."""
    global _lib
    if _lib is not None:
        return _lib
    if _build.variant():
        # an A/B variant is used exactly as built (never silently rebuilt from the
        # current tree, which could make two arms run identical code)
        if not os.path.exists(_build.LIB):
            raise FileNotFoundError(f"ATOS_LIB={_build.LIB} does not exist (build it with ATOS_NVCC_EXTRA first)")
    elif not os.path.exists(_build.LIB) or _build.stale():
        if not build_if_missing:
            raise FileNotFoundError(f"{_build.LIB} missing; run __graft_entry__.build()")
        _build.build()
    lib = ctypes.CDLL(_build.LIB)
    for name, res, args in _SIGS:
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib


def _check(st: int):
    if st != 0:
        raise AtosError(st, load().atos_last_error().decode(errors="replace"))


def default_config(**kw) -> Config:
    cfg = Config()
    _check(load().atos_config_init(ctypes.byref(cfg)))
    for k, v in kw.items():
        if not hasattr(cfg, k):
            raise TypeError(f"unknown atos_config field {k!r}")
        setattr(cfg, k, v)
    return cfg


def partition_balanced(n: int, p: int) -> list:
    part = (ctypes.c_int64 * (p + 1))()
    _check(load().atos_partition_balanced(n, p, part))
    return list(part)


def arena_bytes(n: int, n_ranks: int, rank: int, part=None, **cfg) -> int:
    out = ctypes.c_uint64(0)
    c = default_config(**cfg)
    pa = None
    if part is not None:
        arr = np.ascontiguousarray(part, dtype=np.int64)
        pa = arr.ctypes.data_as(_P)
    _check(load().atos_arena_bytes(n, pa, n_ranks, rank, ctypes.byref(c), ctypes.byref(out)))
    return int(out.value)


def _ptr_of(x):
    """(pointer, keepalive) for numpy arrays or torch tensors (host or device)."""
    if x is None:
        return None, None
    if hasattr(x, "data_ptr"):           # torch tensor
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return ctypes.c_void_p(x.data_ptr()), x
    a = np.ascontiguousarray(x)
    return a.ctypes.data_as(_P), a


class Graph:
    """One rank's (or one process's virtual ranks') view of a loaded graph."""

    def __init__(self, row_ptr, col, n: Optional[int] = None, part: Optional[Sequence[int]] = None, **cfg):
        self._lib = load()
        if hasattr(row_ptr, "dtype") and str(row_ptr.dtype) not in ("int64", "torch.int64"):
            raise TypeError("row_ptr must be int64")
        if hasattr(col, "dtype") and str(col.dtype) not in ("int32", "torch.int32"):
            raise TypeError("col must be int32")
        n = int(n if n is not None else (row_ptr.shape[0] - 1))
        nnz = int(col.shape[0])
        self.n, self.nnz = n, nnz
        self.cfg = default_config(**cfg)
        rp, k1 = _ptr_of(row_ptr)
        cp, k2 = _ptr_of(col)
        pa, k3 = (None, None)
        if part is not None:
            pa, k3 = _ptr_of(np.asarray(part, dtype=np.int64))
        h = ctypes.c_void_p()
        _check(self._lib.atos_graph_load(rp, cp, n, nnz, pa, ctypes.byref(self.cfg), ctypes.byref(h)))
        self._h = h

    # -- multi-process peer mapping --------------------------------------------
    def export_handle(self) -> bytes:
        buf = (ctypes.c_ubyte * ATOS_IPC_HANDLE_BYTES)()
        _check(self._lib.atos_graph_export(self._h, buf))
        return bytes(buf)

    def connect(self, handles: Sequence[bytes]):
        blob = b"".join(handles)
        buf = (ctypes.c_ubyte * len(blob)).from_buffer_copy(blob)
        _check(self._lib.atos_graph_connect(self._h, buf))

    # -- solves ------------------------------------------------------------------
    def bfs(self, src: int, depth_out=None, parent_out=None, parent: bool = False, stats: bool = False):
        """Returns depth (and parent / stats if requested).  Outputs default to numpy
        host arrays; pass torch CUDA tensors to keep them on the device."""
        if depth_out is None:
            depth_out = np.empty(self.n, dtype=np.int32)
        if parent and parent_out is None:
            parent_out = np.empty(self.n, dtype=np.int64)
        dp, _k1 = _ptr_of(depth_out)
        pp, _k2 = _ptr_of(parent_out)
        st = Stats() if stats else None
        _check(self._lib.atos_bfs(self._h, int(src), dp, pp, ctypes.byref(st) if st is not None else None))
        out = [depth_out]
        if parent_out is not None:
            out.append(parent_out)
        if st is not None:
            out.append(st.as_dict())
        return out[0] if len(out) == 1 else tuple(out)

    def pagerank(self, alpha: float = 0.85, eps: float = 1e-9, rank_out=None, residual_out=None,
                 stats: bool = False):
        if rank_out is None:
            rank_out = np.empty(self.n, dtype=np.float64)
        if residual_out is None:
            residual_out = np.empty(self.n, dtype=np.float64)
        rp, _k1 = _ptr_of(rank_out)
        sp, _k2 = _ptr_of(residual_out)
        st = Stats() if stats else None
        _check(self._lib.atos_pagerank(self._h, float(alpha), float(eps), rp, sp,
                                       ctypes.byref(st) if st is not None else None))
        if st is not None:
            return rank_out, residual_out, st.as_dict()
        return rank_out, residual_out

    def set_watchdog(self, ms: int):
        _check(self._lib.atos_set_watchdog(self._h, int(ms)))

    def sync(self):
        _check(self._lib.atos_sync(self._h))

    def last_stats(self) -> dict:
        st = Stats()
        _check(self._lib.atos_last_stats(self._h, ctypes.byref(st)))
        return st.as_dict()

    def free(self):
        if getattr(self, "_h", None):
            self._lib.atos_graph_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()


QB_OPS = {"push": 0, "pop": 1, "push_then_pop": 2}


def queue_bench(worker_size: int, op: str, threads: int, rounds: int = 10, fetch_size: Optional[int] = None,
                ring_cap: Optional[int] = None, index_base: int = 0, reserve_cas: bool = False,
                popped: bool = False, device: int = 0):
    """atos_queue_bench: returns (ms, popped items or None)."""
    total = threads * rounds
    if ring_cap is None:
        ring_cap = 1 << max(10, (total - 1).bit_length())
    c = QBenchConfig(worker_size, fetch_size or worker_size, QB_OPS[op], rounds, threads, ring_cap, index_base,
                     1 if reserve_cas else 0, device)
    out = np.empty(total, dtype=np.uint32) if popped else None
    ms = ctypes.c_double(0)
    _check(load().atos_queue_bench(ctypes.byref(c), out.ctypes.data_as(_P) if out is not None else None,
                                   ctypes.byref(ms)))
    return ms.value, out


# function-style aliases with the C names
def graph_load(row_ptr, col, n=None, part=None, **cfg) -> Graph:
    return Graph(row_ptr, col, n, part, **cfg)


def bfs(g: Graph, src: int, **kw):
    return g.bfs(src, **kw)


def pagerank(g: Graph, alpha: float, eps: float, **kw):
    return g.pagerank(alpha, eps, **kw)


def graph_free(g: Graph):
    g.free()

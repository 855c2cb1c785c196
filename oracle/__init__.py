"""CPU oracle for the Atos hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(paper_conf_sc_chenbpbyo22_b200) never imports it and shares no code with it.

Functions (see oracle.c for the paper passages each one follows):
  bfs(row_ptr, col, src)                -> depth int32 [n]   (-1 = unreachable)
  bfs_parents_minid(row_ptr, col, depth, src) -> parent int64 [n]
  pagerank(row_ptr, col, alpha, tol)    -> (p float64 [n] with sum 1, iterations, final L1 delta);
                                           raises RuntimeError if max_iter ends before ||dp||_1 <= tol

Parity status: BFS pinned (brute force / closed forms / scipy); PageRank pinned
(closed forms / dense solve / networkx).  See tests/test_oracle.py.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "_oracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c -> oracle/_oracle.so with plain gcc (+OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        p = ctypes.c_void_p
        i64 = ctypes.c_int64
        lib.oracle_bfs.argtypes = [i64, p, p, i64, p]
        lib.oracle_bfs_parents_minid.argtypes = [i64, p, p, p, i64, p]
        lib.oracle_pagerank.argtypes = [i64, p, p, ctypes.c_double, ctypes.c_double, ctypes.c_int,
                                        ctypes.c_int, p, p, p]
        for f in (lib.oracle_bfs, lib.oracle_bfs_parents_minid, lib.oracle_pagerank):
            f.restype = ctypes.c_int
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _np(x, dtype):
    if hasattr(x, "detach"):          # torch tensor
        x = x.detach().cpu().numpy()
    return np.ascontiguousarray(x, dtype=dtype)


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def bfs(row_ptr, col, src: int) -> np.ndarray:
    rp = _np(row_ptr, np.int64)
    c = _np(col, np.int32)
    n = rp.size - 1
    depth = np.empty(n, dtype=np.int32)
    rc = _load().oracle_bfs(n, _ptr(rp), _ptr(c), int(src), _ptr(depth))
    if rc != 0:
        raise ValueError(f"oracle_bfs failed rc={rc}")
    return depth


def bfs_parents_minid(row_ptr, col, depth, src: int) -> np.ndarray:
    rp = _np(row_ptr, np.int64)
    c = _np(col, np.int32)
    d = _np(depth, np.int32)
    n = rp.size - 1
    parent = np.empty(n, dtype=np.int64)
    rc = _load().oracle_bfs_parents_minid(n, _ptr(rp), _ptr(c), _ptr(d), int(src), _ptr(parent))
    if rc != 0:
        raise ValueError(f"oracle_bfs_parents_minid failed rc={rc}")
    return parent


def pagerank(row_ptr, col, alpha: float = 0.85, tol: float = 1e-12, max_iter: int = 10000,
             nthreads: int = 0):
    rp = _np(row_ptr, np.int64)
    c = _np(col, np.int32)
    n = rp.size - 1
    p = np.empty(n, dtype=np.float64)
    it = ctypes.c_int(0)
    delta = ctypes.c_double(0.0)
    rc = _load().oracle_pagerank(n, _ptr(rp), _ptr(c), float(alpha), float(tol), int(max_iter),
                                 int(nthreads), _ptr(p), ctypes.byref(it), ctypes.byref(delta))
    if rc == 4:
        raise RuntimeError(f"oracle_pagerank did not converge: ||dp||_1 = {delta.value:.3e} > tol {tol:.1e} "
                           f"after {it.value} iterations (max_iter {max_iter})")
    if rc != 0:
        raise ValueError(f"oracle_pagerank failed rc={rc}")
    return p, it.value, delta.value

"""Seeded synthetic graph inputs shared by the CUDA path and the oracle.

This module holds NO arithmetic of the method (no traversal, no relaxation,
no PageRank step).  It only draws graphs: a counter-based splitmix64 stream,
Graph500-style Kronecker/RMAT edge generation, a keyed label bijection, a
road-like 2-D grid, CSR assembly, and BFS source sampling.  Both sides of every
parity test receive the same CSR from here; neither side imports the other.

Everything is written with plain torch integer ops so that the CPU and the GPU
draw bit-identical graphs (checked in tests/test_inputs.py against a numpy
uint64 re-implementation of splitmix64).

Workload shapes follow the paper's datasets (Table I:
scale-free social graphs with skewed degree; mesh-like road graphs with avg
degree ~2.5 and diameter in the thousands) and BASELINE.json `configs`.
The recipe is written out in DESIGN.md §3 (readings #10-#12 of SURVEY §8c).
"""
from __future__ import annotations

import dataclasses
import math
from typing import List, Optional

import torch

# --------------------------------------------------------------------------
# splitmix64 on torch.int64 (two's complement wrap-around == uint64 arithmetic)
# --------------------------------------------------------------------------
_M64 = (1 << 64)


def _s64(x: int) -> int:
    """Map an unsigned 64-bit constant to the signed int64 with the same bits."""
    x &= _M64 - 1
    return x - _M64 if x >= (1 << 63) else x


_GAMMA = _s64(0x9E3779B97F4A7C15)
_MIX1 = _s64(0xBF58476D1CE4E5B9)
_MIX2 = _s64(0x94D049BB133111EB)


def _lsr(z: torch.Tensor, k: int) -> torch.Tensor:
    """Logical shift right of int64 bit patterns."""
    return (z >> k) & ((1 << (64 - k)) - 1)


def _mix64(z: torch.Tensor) -> torch.Tensor:
    z = (z ^ _lsr(z, 30)) * _MIX1
    z = (z ^ _lsr(z, 27)) * _MIX2
    return z ^ _lsr(z, 31)


def _key(seed: int, stream: int) -> int:
    """Per-(seed, stream) base state of the counter-based generator (python int)."""
    t = torch.tensor([_s64(seed * 0x100000001B3 + stream)], dtype=torch.int64)
    return int(_mix64(t + _GAMMA)[0])


def splitmix64(key: int, counter: torch.Tensor) -> torch.Tensor:
    """The counter-th output of splitmix64 started at state `key` (int64 bits)."""
    return _mix64(key + (counter + 1) * _GAMMA)


def uniform53(key: int, counter: torch.Tensor) -> torch.Tensor:
    """U[0,1) with 53 random bits, exactly representable in fp64."""
    return _lsr(splitmix64(key, counter), 11).to(torch.float64) * (2.0 ** -53)


# --------------------------------------------------------------------------
# CSR container
# --------------------------------------------------------------------------
@dataclasses.dataclass
class CSR:
    """Directed out-edge CSR: row_ptr int64 [n+1], col int32 [nnz] (global ids)."""
    n: int
    row_ptr: torch.Tensor
    col: torch.Tensor
    name: str = ""
    symmetric: bool = False

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    def to(self, device) -> "CSR":
        return CSR(self.n, self.row_ptr.to(device), self.col.to(device), self.name, self.symmetric)

    def numpy(self):
        return self.row_ptr.cpu().numpy(), self.col.cpu().numpy()

    def degrees(self) -> torch.Tensor:
        return self.row_ptr[1:] - self.row_ptr[:-1]


def csr_from_edges(n: int, src: torch.Tensor, dst: torch.Tensor, *, symmetrize: bool,
                   drop_self_loops: bool = True, dedup: bool = True, name: str = "") -> CSR:
    """Assemble a CSR sorted by (src, dst).  Multiplicity is kept iff dedup=False."""
    src = src.to(torch.int64)
    dst = dst.to(torch.int64)
    if drop_self_loops:
        keep = src != dst
        src, dst = src[keep], dst[keep]
    if symmetrize:
        src, dst = torch.cat([src, dst]), torch.cat([dst, src])
    key = src * n + dst
    del src, dst
    if dedup:
        key = torch.unique(key, sorted=True)
    else:
        key, _ = torch.sort(key)
    s = torch.div(key, n, rounding_mode="floor")
    col = (key - s * n).to(torch.int32)
    del key
    counts = torch.bincount(s, minlength=n)
    del s
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=col.device)
    torch.cumsum(counts, 0, out=row_ptr[1:])
    return CSR(n, row_ptr, col, name, symmetrize)


def csr_from_lists(adj: List[List[int]], name: str = "") -> CSR:
    """Tiny hand-written graphs for tests: adj[v] = out-neighbour list (kept as given)."""
    n = len(adj)
    row_ptr = [0]
    col = []
    for nb in adj:
        col.extend(nb)
        row_ptr.append(len(col))
    return CSR(n, torch.tensor(row_ptr, dtype=torch.int64), torch.tensor(col, dtype=torch.int32), name)


# --------------------------------------------------------------------------
# Kronecker / RMAT (Graph500 semantics, no noise)
# --------------------------------------------------------------------------
RMAT_ABCD = (0.57, 0.19, 0.19, 0.05)


def _label_bijection(x: torch.Tensor, scale: int, seed: int) -> torch.Tensor:
    """Keyed bijection on [0, 2^scale): 4 rounds of (odd-multiply-add, xorshift)."""
    mask = (1 << scale) - 1
    h = max(1, (scale + 1) // 2)
    for r in range(4):
        k = int(splitmix64(_key(seed, 0x5EED + r), torch.tensor([0]))[0]) & ((1 << 62) - 1)
        a = ((k >> 20) & mask) | 1
        b = k & mask
        x = (x * a + b) & mask        # x < 2^scale <= 2^31, a < 2^31: no overflow
        x = x ^ (x >> h)
    return x


def rmat_edges(scale: int, edgefactor: int, seed: int, device="cpu", permute: bool = True,
               chunk: int = 1 << 25):
    """m = edgefactor * 2^scale generated edges (src, dst) as int64 tensors."""
    A, B, C, D = RMAT_ABCD
    ab = A + B
    c_norm = C / (C + D)
    a_norm = A / (A + B)
    m = edgefactor * (1 << scale)
    key = _key(seed, 0x52AA7)
    srcs, dsts = [], []
    for lo in range(0, m, chunk):
        hi = min(m, lo + chunk)
        i = torch.arange(lo, hi, dtype=torch.int64, device=device)
        s = torch.zeros_like(i)
        d = torch.zeros_like(i)
        for b in range(scale):
            base = (i * scale + b) * 2
            u1 = uniform53(key, base)
            u2 = uniform53(key, base + 1)
            row_bit = u1 > ab
            col_bit = torch.where(row_bit, u2 > c_norm, u2 > a_norm)
            s = s | (row_bit.to(torch.int64) << b)
            d = d | (col_bit.to(torch.int64) << b)
        if permute:
            s = _label_bijection(s, scale, seed)
            d = _label_bijection(d, scale, seed)
        srcs.append(s)
        dsts.append(d)
    return torch.cat(srcs), torch.cat(dsts)


def rmat(scale: int, edgefactor: int = 16, seed: int = 1, *, symmetric: bool, permute: bool = True,
         device="cpu") -> CSR:
    s, d = rmat_edges(scale, edgefactor, seed, device=device, permute=permute)
    kind = "sym" if symmetric else "dir"
    name = f"{'rmat' if permute else 'kron'}{scale}_ef{edgefactor}_{kind}_s{seed}"
    return csr_from_edges(1 << scale, s, d, symmetrize=symmetric, name=name)


# --------------------------------------------------------------------------
# Road-like grid (road_usa shape)
# --------------------------------------------------------------------------
def road_grid(W: int = 4900, H: int = 4900, seed: int = 1, p_vertical: float = 0.25,
              device="cpu") -> CSR:
    """All horizontal edges; vertical edge (r,c)-(r+1,c) kept iff U < p_vertical; symmetric."""
    n = W * H
    key = _key(seed, 0x60AD)
    r = torch.arange(H, dtype=torch.int64, device=device).repeat_interleave(W - 1)
    c = torch.arange(W - 1, dtype=torch.int64, device=device).repeat(H)
    hs = r * W + c
    hd = hs + 1
    rv = torch.arange(H - 1, dtype=torch.int64, device=device).repeat_interleave(W)
    cv = torch.arange(W, dtype=torch.int64, device=device).repeat(H - 1)
    vid = rv * W + cv
    keep = uniform53(key, vid) < p_vertical
    vs = vid[keep]
    vd = vs + W
    src = torch.cat([hs, vs])
    dst = torch.cat([hd, vd])
    return csr_from_edges(n, src, dst, symmetrize=True, name=f"grid{W}x{H}_s{seed}")


# --------------------------------------------------------------------------
# Sources, partitions
# --------------------------------------------------------------------------
def bfs_sources(g: CSR, count: int, seed: int = 1) -> List[int]:
    """`count` distinct non-isolated sources drawn from the seeded stream (Graph500 style)."""
    deg = g.degrees().cpu()
    key = _key(seed, 0x50C)
    out: List[int] = []
    k = 0
    while len(out) < count and k < 64 * count + 1024:
        v = int(_lsr(splitmix64(key, torch.tensor([k])), 1)[0] % g.n)
        k += 1
        if deg[v] > 0 and v not in out:
            out.append(v)
    return out


def balanced_partition(n: int, p: int) -> List[int]:
    """1-D contiguous vertex blocks: part[r] = floor(r*n/p)  (reading #13)."""
    return [(r * n) // p for r in range(p + 1)]


# --------------------------------------------------------------------------
# BASELINE.json configs as concrete instances
# --------------------------------------------------------------------------
CONFIGS = {
    # configs[0]: BFS from vertex 0, Kronecker scale-12 ef16 (unpermuted: vertex 0 is the hub)
    "kron12": dict(kind="rmat", scale=12, edgefactor=16, symmetric=True, permute=False, app="bfs"),
    # configs[1]: async PageRank alpha=.85 eps=1e-9, RMAT-20 ef16 directed
    "rmat20_pr": dict(kind="rmat", scale=20, edgefactor=16, symmetric=False, permute=True, app="pr"),
    # configs[2]: BFS RMAT-24 ef16 (symmetrised), 1/2/4/8 GPUs
    "rmat24": dict(kind="rmat", scale=24, edgefactor=16, symmetric=True, permute=True, app="bfs"),
    # configs[3]: road-like grid, ~24M vertices, avg deg ~2.5
    "grid4900": dict(kind="grid", W=4900, H=4900, app="bfs"),
    # configs[4]: PageRank RMAT-26 directed across 8 GPUs
    "rmat26_pr": dict(kind="rmat", scale=26, edgefactor=16, symmetric=False, permute=True, app="pr"),
    # north_star target: BFS RMAT-26 symmetric
    "rmat26": dict(kind="rmat", scale=26, edgefactor=16, symmetric=True, permute=True, app="bfs"),
    # quick-check size for multi-process smoke runs (not a BASELINE config)
    "rmat18": dict(kind="rmat", scale=18, edgefactor=16, symmetric=True, permute=True, app="bfs"),
}


def make_config(name: str, seed: int = 1, device="cpu", **override) -> CSR:
    cfg = dict(CONFIGS[name])
    cfg.update(override)
    if cfg["kind"] == "rmat":
        g = rmat(cfg["scale"], cfg["edgefactor"], seed, symmetric=cfg["symmetric"],
                 permute=cfg["permute"], device=device)
    else:
        g = road_grid(cfg["W"], cfg["H"], seed, device=device)
    if str(device).startswith("cuda"):
        # the generator's temporaries (edge lists, sort buffers: tens of GB at
        # scale 26) stay in torch's cache otherwise, and libatos allocates with
        # cudaMalloc outside that cache
        torch.cuda.empty_cache()
    return g

"""GPU: per-iteration cost of the discrete-kernel mode on a path (one vertex per launch)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs
n = 2000
idx = torch.arange(n - 1, device="cuda")
g = inputs.csr_from_edges(n, idx, idx + 1, symmetrize=True, name="path")
for cfg in ({"discrete": 1, "keep_items": 0}, {"discrete": 1, "keep_items": 0, "l2_persist": 0},
            {"discrete": 1, "keep_items": 0, "ctas_per_sm": 1}, {"keep_items": 0}, {"keep_items": 0, "l2_persist": 0}):
    G = atos.Graph(g.row_ptr, g.col, g.n, **cfg)
    d = torch.empty(n, dtype=torch.int32, device="cuda")
    for _ in range(2):
        G.bfs(0, depth_out=d); st = G.last_stats()
    print(cfg, "ms_worker %.3f  us/level %.2f  iterations %d" % (st["ms_worker"], st["ms_worker"] * 1e3 / n, st["iterations"]), flush=True)
    G.free()

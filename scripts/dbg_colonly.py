import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs
g = inputs.make_config("rmat24", device="cuda")
G = atos.Graph(g.row_ptr, g.col, g.n)
# diagnostic build: each BFS only expands the source's batch chain; use many sources
d = torch.empty(g.n, dtype=torch.int32, device="cuda")
for s in inputs.bfs_sources(g, 3):
    G.bfs(s, depth_out=d); st = G.last_stats(); print(st["ms_worker"], st["edges"], flush=True)

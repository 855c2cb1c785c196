import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs
g = inputs.make_config("kron12")
rp, col = g.numpy()
cfg = dict(relabel=int(sys.argv[1]), hub_cache=int(sys.argv[2]))
with atos.Graph(rp, col, **cfg) as G:
    d = G.bfs(0)
print("ok", cfg, (d >= 0).sum())

import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs
for scale in [int(x) for x in sys.argv[1].split(",")]:
    g = inputs.rmat(scale, 16, 1, symmetric=True, device="cuda")
    G = atos.Graph(g.row_ptr, g.col, g.n, watchdog_ms=20000)
    rp, col = g.numpy()
    for s in inputs.bfs_sources(g, 3):
        try:
            d = G.bfs(s)
            ok = np.array_equal(d, oracle.bfs(rp, col, s))
            print(scale, s, "ok" if ok else "MISMATCH", G.last_stats()["ms_worker"], flush=True)
        except Exception as e:
            print(scale, s, "ERR", e, flush=True); break
    G.free()

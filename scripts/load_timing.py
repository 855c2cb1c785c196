"""GPU: wall time of atos_graph_load + one BFS + free from pinned host / device CSR, relabel on/off."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs

g = inputs.make_config(sys.argv[1] if len(sys.argv) > 1 else "rmat24", device="cuda")
rp_h, col_h = g.row_ptr.cpu().pin_memory(), g.col.cpu().pin_memory()
d_h = torch.empty(g.n, dtype=torch.int32).pin_memory()
src = inputs.bfs_sources(g, 1)[0]
for where in ("host", "device"):
    for rl in (0, 2):
        for rep in range(2):
            rp, col = (rp_h, col_h) if where == "host" else (g.row_ptr, g.col)
            torch.cuda.synchronize(); t0 = time.perf_counter()
            G = atos.Graph(rp, col, g.n, relabel=rl)
            torch.cuda.synchronize(); t1 = time.perf_counter()
            G.bfs(src, depth_out=d_h); G.sync()
            t2 = time.perf_counter()
            G.free(); torch.cuda.synchronize(); t3 = time.perf_counter()
            print(f"{where:6s} relabel={rl} load {1e3*(t1-t0):8.1f} ms  bfs+d2h {1e3*(t2-t1):7.1f} ms  free {1e3*(t3-t2):7.1f} ms", flush=True)

"""GPU: bench.py's e2e loop (load from pinned host CSR + BFS to host + free) with the load trace."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs
g = inputs.make_config("rmat24", device="cuda")
stream = torch.cuda.current_stream()
cfg = dict(agg_enabled=1, stream=stream.cuda_stream)
G = atos.Graph(g.row_ptr, g.col, g.n, **cfg)
src = inputs.bfs_sources(g, 1)[0]
rp_h, col_h = g.row_ptr.cpu().pin_memory(), g.col.cpu().pin_memory()
d_h = torch.empty(g.n, dtype=torch.int32).pin_memory()
print("stream handle", stream.cuda_stream, flush=True)
for k in range(4):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    H = atos.Graph(rp_h, col_h, g.n, **cfg)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    H.bfs(src, depth_out=d_h)
    t2 = time.perf_counter()
    H.free(); torch.cuda.synchronize(); t3 = time.perf_counter()
    print(f"load {1e3*(t1-t0):.1f} ms  bfs {1e3*(t2-t1):.1f} ms  free {1e3*(t3-t2):.1f} ms", flush=True)

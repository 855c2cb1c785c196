"""Lean driver for ncu: generate + load + warm up outside the profiled range, then
profile exactly one solve (run ncu with --profile-from-start off)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_chenbpbyo22_b200 import atos, inputs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--app", default="bfs", choices=["bfs", "pr"])
    ap.add_argument("--graph", default=None)
    ap.add_argument("--solves", type=int, default=1)
    ap.add_argument("--cfg", default="{}", help="atos_config overrides (JSON)")
    args = ap.parse_args()
    name = args.graph or ("rmat24" if args.app == "bfs" else "rmat20_pr")
    g = inputs.make_config(name, device="cuda")
    stream = torch.cuda.current_stream()
    import json
    G = atos.Graph(g.row_ptr, g.col, g.n, stream=stream.cuda_stream, **json.loads(args.cfg))
    if args.app == "bfs":
        srcs = [0] if name == "kron12" else inputs.bfs_sources(g, 4)
        depth = torch.empty(g.n, dtype=torch.int32, device="cuda")
        for s in srcs[:3]:
            G.bfs(s, depth_out=depth)
            G.sync()
        torch.cuda.synchronize()
        torch.cuda.profiler.start()
        for i in range(args.solves):
            G.bfs(srcs[3 % len(srcs)], depth_out=depth)
            G.sync()
        torch.cuda.profiler.stop()
    else:
        r = torch.empty(g.n, dtype=torch.float64, device="cuda")
        s_ = torch.empty(g.n, dtype=torch.float64, device="cuda")
        for _ in range(2):
            G.pagerank(0.85, 1e-9, rank_out=r, residual_out=s_)
            G.sync()
        torch.cuda.synchronize()
        torch.cuda.profiler.start()
        for i in range(args.solves):
            G.pagerank(0.85, 1e-9, rank_out=r, residual_out=s_)
            G.sync()
        torch.cuda.profiler.stop()
    print(G.last_stats())
    G.free()


if __name__ == "__main__":
    main()

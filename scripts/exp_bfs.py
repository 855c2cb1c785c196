"""Exploration harness (GPU): BFS worker timing + counters under several configs."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_chenbpbyo22_b200 import atos, inputs  # noqa: E402


def run(g, srcs, reps=4, **cfg):
    G = atos.Graph(g.row_ptr, g.col, g.n, **cfg)
    depth = torch.empty(g.n, dtype=torch.int32, device="cuda")
    deg = g.degrees()
    rows = []
    for i in range(reps + 1):
        s = srcs[i % len(srcs)]
        G.bfs(s, depth_out=depth)
        st = G.last_stats()
        if i == 0:
            continue
        reached = depth >= 0
        m = int(deg[reached].sum())
        nr = int(reached.sum())
        util = st["busy_ns"] / max(1e-9, st["grid_ctas"] * st["n_ranks"] * st["ms_worker"] * 1e6)
        rows.append(dict(ms=st["ms_worker"], gteps=m / st["ms_worker"] / 1e6, pops=st["pops"] / nr,
                         edges=st["edges"] / m, util=util, batches=st["batches"], idle=st["idle_polls"], iters=st["iterations"],
                         hub=st["hub_hits"] / max(1, st["edges"]), msgs=st["msgs_sent"],
                         mpp=st["msgs_sent"] / max(1, st["packets_sent"])))
    G.free()
    agg = {k: sum(r[k] for r in rows) / len(rows) for k in rows[0]}
    return agg


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graph", default="rmat24")
    ap.add_argument("--configs", default='[{}]')
    args = ap.parse_args()
    try:
        from cuda.bindings import runtime as cudart
        _, p = cudart.cudaGetDeviceProperties(0)
        print(f"persistingL2CacheMaxSize={p.persistingL2CacheMaxSize} accessPolicyMaxWindowSize="
              f"{p.accessPolicyMaxWindowSize} l2={p.l2CacheSize}", flush=True)
    except Exception as e:  # pragma: no cover
        print("props unavailable:", e)
    t0 = time.time()
    if args.graph.startswith("path"):
        n = int(args.graph[4:])
        idx = torch.arange(n - 1, device="cuda")
        g = inputs.csr_from_edges(n, idx, idx + 1, symmetrize=True)
        srcs = [0]
    else:
        import re
        m = re.fullmatch(r"rmat(\d+)", args.graph)
        if m and args.graph not in inputs.CONFIGS:      # any RMAT scale, configs[2]'s recipe
            g = inputs.make_config("rmat24", device="cuda", scale=int(m.group(1)))
        else:
            g = inputs.make_config(args.graph, device="cuda")
        srcs = [0] if args.graph in ("kron12", "grid4900") else inputs.bfs_sources(g, 8)
    print(f"graph {g.name} n={g.n} nnz={g.nnz} gen {time.time()-t0:.1f}s", flush=True)
    for cfg in json.loads(args.configs):
        r = run(g, srcs, **cfg)
        print(json.dumps({"cfg": cfg, **{k: round(v, 4) for k, v in r.items()}}), flush=True)


if __name__ == "__main__":
    main()

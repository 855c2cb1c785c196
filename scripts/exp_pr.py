"""Exploration harness (GPU): PageRank worker timing + counters under several configs."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_chenbpbyo22_b200 import atos, inputs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graph", default="rmat20_pr")
    ap.add_argument("--configs", default='[{}]')
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    g = inputs.make_config(args.graph, device="cuda")
    print(f"graph {g.name} n={g.n} nnz={g.nnz}", flush=True)
    r = torch.empty(g.n, dtype=torch.float64, device="cuda")
    s = torch.empty(g.n, dtype=torch.float64, device="cuda")
    for cfg in json.loads(args.configs):
        P = atos.Graph(g.row_ptr, g.col, g.n, **cfg)
        rows = []
        for i in range(args.reps + 1):
            P.pagerank(0.85, 1e-9, rank_out=r, residual_out=s)
            st = P.last_stats()
            if i:
                rows.append(st)
        P.free()
        ms = sum(x["ms_worker"] for x in rows) / len(rows)
        rel = sum(x["edges"] for x in rows) / len(rows)
        pops = sum(x["pops"] for x in rows) / len(rows)
        msgs = sum(x["msgs_sent"] for x in rows) / len(rows)
        iters = sum(x["iterations"] for x in rows) / len(rows)
        pk = sum(x["packets_sent"] for x in rows) / len(rows)
        print(json.dumps({"cfg": cfg, "ms": round(ms, 3), "relax_per_nnz": round(rel / g.nnz, 2),
                          "pops_per_v": round(pops / g.n, 2), "gatomics": round(rel / ms / 1e6, 1),
                          "msgs_M": round(msgs / 1e6, 2), "packets_K": round(pk / 1e3, 2),
                          "msg_GBps": round(msgs * 16 / ms / 1e6, 1), "iters": iters}), flush=True)


if __name__ == "__main__":
    main()

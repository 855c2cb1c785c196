"""Real multi-process path (IPC export/connect, cross-process barrier, coordinator,
one-sided channel stores) with every rank on the SAME GPU -- the only multi-process
configuration a 1-GPU box can run.  The contexts are time-sliced, so it checks the
protocol, not the speed.

    python -m torch.distributed.run --standalone --nproc-per-node 2 scripts/mp_same_gpu.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import oracle  # noqa: E402
from paper_conf_sc_chenbpbyo22_b200 import atos, inputs  # noqa: E402
from paper_conf_sc_chenbpbyo22_b200 import dist as adist  # noqa: E402


def main():
    rank, world, _ = adist.init(backend="gloo")
    torch.cuda.set_device(0)
    ok = True
    scale = int(os.environ.get("ATOS_MP_SCALE", "13"))
    g = inputs.rmat(scale, 16, 1, symmetric=True)
    rp, col = g.numpy()
    G = atos.Graph(rp, col, g.n, rank=rank, n_ranks=world, device=0, ctas_per_sm=1, watchdog_ms=600000,
                   channel_packets=64)
    adist.connect_graph(G, world)
    dist.barrier()
    for s in inputs.bfs_sources(g, 2):
        d, par, st = G.bfs(s, parent=True, stats=True)
        want = oracle.bfs(rp, col, s)
        good = np.array_equal(d, want) and np.array_equal(par, oracle.bfs_parents_minid(rp, col, want, s))
        ok &= good
        print(f"[rank {rank}] bfs src={s} {'ok' if good else 'MISMATCH'} msgs={st['msgs_sent']} "
              f"packets={st['packets_sent']} ms={st['ms_worker']:.1f}", flush=True)
        dist.barrier()
    G.free()
    gd = inputs.rmat(scale - 1, 16, 2, symmetric=False)
    rp, col = gd.numpy()
    P = atos.Graph(rp, col, gd.n, rank=rank, n_ranks=world, device=0, ctas_per_sm=1, watchdog_ms=600000,
                   channel_packets=64)
    adist.connect_graph(P, world)
    dist.barrier()
    rank_out, res_out, st = P.pagerank(0.85, 1e-9, stats=True)
    p, _, _ = oracle.pagerank(rp, col, 0.85, 1e-12)
    err = np.abs(rank_out / rank_out.sum() - p)
    good = err.max() <= 1e-6 and err.sum() <= 1e-5 and np.all(res_out < 1e-9)
    ok &= good
    print(f"[rank {rank}] pagerank {'ok' if good else 'MISMATCH'} L1={err.sum():.2e} msgs={st['msgs_sent']}",
          flush=True)
    dist.barrier()
    P.free()
    okt = torch.tensor([1 if ok else 0])
    dist.all_reduce(okt, op=dist.ReduceOp.MIN)
    if rank == 0:
        print("MP_SAME_GPU", "PASS" if okt.item() == 1 else "FAIL", flush=True)
    dist.destroy_process_group()
    sys.exit(0 if okt.item() == 1 else 1)


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""bench.py -- BFS & PageRank GTEPS of the B200-native Atos hot path.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl atos|reference] [--workload NAME]

Headline (BASELINE.json metric, configs[2]): asynchronous push BFS on RMAT-24
ef16 (symmetrised), 1-D vertex partition over N GPUs (strong scaling), one step
= one BFS solve (barrier, init, persistent worker, termination, gather) from
the next of 16 sampled non-isolated sources.  value = sum of m_reached over the
K timed steps / device time (max over ranks), in GTEPS, m_reached = directed
CSR entries of reached vertices (reading R23).  The PageRank line of
the metric (configs[1], RMAT-20 directed, alpha .85, eps 1e-9) is reported
under "pagerank".  Inputs are seeded synthetic graphs generated on the device;
the CSR (2.2 GB) is larger than L2 (126 MB), so no L2 flush is done between
steps (said in config.l2).

--impl reference times the CPU oracle (oracle/, test infrastructure) on the
same workload: each step is one serial BFS from that step's source.

--gpus N without a torchrun environment re-launches itself under
torch.distributed.run with N ranks (one process per GPU, 127.0.0.1
rendezvous); on a box with fewer than N GPUs the ranks share device 0
(ATOS_SAME_DEVICE, time-sliced: a protocol check, not a scaling number, and the
line says so in config.same_device).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_chenbpbyo22_b200 import dist as adist  # noqa: E402
from paper_conf_sc_chenbpbyo22_b200 import inputs  # noqa: E402

WORKLOADS = {
    "bfs_rmat24": ("rmat24", "bfs"),
    "bfs_rmat26": ("rmat26", "bfs"),
    "bfs_kron12": ("kron12", "bfs"),
    "bfs_grid4900": ("grid4900", "bfs"),
    "bfs_rmat18": ("rmat18", "bfs"),      # quick-check size (not a BASELINE config)
}
KERNELS_PER_BFS_STEP = {1: 5}    # init, seed, worker, fixup, gather (+ barrier when N > 1)


METRIC = "BFS & PageRank GTEPS (max over ranks); headline = BFS GTEPS"


def arm_config(args, g, srcs, world):
    """The `config` object both arms report (same workload, same keys)."""
    return {"workload": args.workload, "graph": g.name, "n": g.n, "nnz": g.nnz,
            "sources": len(srcs), "partition": "1d-balanced", "parallelism": f"vertex-1d x{world}",
            "aggregation": bool(args.agg),
            "vertex_order": "degree-relabeled inside rank blocks (atos_config.relabel=auto); outputs in generator ids",
            "queue": ("one rank: level buckets (N1 priority queue, threshold_delta 1; atos_config.pq_delta=auto) "
                      "with an n-bit visited bitmap and claim at pop; several ranks: FIFO queue with the "
                      "u8 depth-bound filter (atos_config.probe_filter=auto)"),
            "l2": ("no flush: CSR inputs larger than L2 (%.2f GB > 126 MB)" % ((g.nnz * 4 + g.n * 8) / 1e9))
            if g.nnz * 4 + g.n * 8 > 126e6 else "CSR fits L2 (%.1f MB): a latency figure, not a bandwidth one"
                                                % ((g.nnz * 4 + g.n * 8) / 1e6)}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def micro_peak(key):
    """A denominator measured by scripts/micro.cu on this pool's B200 (committed under profiles/)."""
    p = os.path.join(ROOT, "profiles", "r1", "micro_denominators.json")
    try:
        return float(json.load(open(p))[key])
    except Exception:
        return None


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, STREAM-style copy)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.3)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        self.lines = []
        if self.proc is not None:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                out, _ = self.proc.communicate(timeout=5)
            except Exception:
                self.proc.kill()
                out = ""
            self.lines = [l for l in out.splitlines() if l.strip()]

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in getattr(self, "lines", []):
            f = [x.strip() for x in l.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


def make_graph(name: str, device):
    t0 = time.time()
    g = inputs.make_config(name, device=device)
    log(f"[bench] generated {g.name}: n={g.n} nnz={g.nnz} in {time.time() - t0:.1f}s on {device}")
    return g


def m_reached_of(depth_dev: torch.Tensor, deg: torch.Tensor):
    reached = depth_dev >= 0
    return int(deg[reached].sum().item()), int(reached.sum().item())


def cpu_baseline_bfs(g, src: int, m_reached: int):
    import oracle
    rp, col = g.row_ptr.cpu().numpy(), g.col.cpu().numpy()
    t0 = time.perf_counter()
    d = oracle.bfs(rp, col, src)
    dt = time.perf_counter() - t0
    return {"value": m_reached / dt / 1e9, "unit": "GTEPS", "cores": 1, "kind": "oracle",
            "sample": f"1 serial FIFO BFS (oracle/oracle.c) from source {src} on the full {g.name} graph, "
                      f"{dt:.2f} s on 1 host core", "seconds": dt, "reached": int((d >= 0).sum())}


def run_reference(args, rank, world):
    """Reference arm = the CPU oracle, timed as it stands on the box's host cores."""
    if rank != 0:
        return
    import oracle
    gname, app = WORKLOADS[args.workload]
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    g = make_graph(gname, dev)
    srcs = [0] if gname == "kron12" else inputs.bfs_sources(g, args.sources)
    rp, col = g.row_ptr.cpu().numpy(), g.col.cpu().numpy()
    deg = np.diff(rp)
    for k in range(args.warmup):
        oracle.bfs(rp, col, srcs[k % len(srcs)])
    edges = 0
    t0 = time.perf_counter()
    for k in range(args.steps):
        d = oracle.bfs(rp, col, srcs[(args.warmup + k) % len(srcs)])
        edges += int(deg[d >= 0].sum())
    dt = time.perf_counter() - t0
    v = edges / dt / 1e9
    line = {"impl": "reference", "metric": METRIC,
            "value": v, "unit": "GTEPS", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": dt * 1e3 / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "i32", "data": "synthetic (seeded Graph500 RMAT)",
            "config": arm_config(args, g, srcs, world),
            "cpu_baseline": {"value": v, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                             "sample": f"{args.steps} serial FIFO BFS solves (oracle/oracle.c) on the full graph"},
            "e2e": {"value": v, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def spawn(n: int) -> int:
    """Re-launch this command as n ranks under torch.distributed.run (one node)."""
    import socket
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    try:
        ndev = torch.cuda.device_count()
    except Exception:
        ndev = 0
    if ndev < n:
        env["ATOS_SAME_DEVICE"] = "1"      # every rank on device 0 (time-sliced protocol check)
        log(f"[bench] {ndev} GPU(s) visible for --gpus {n}: ranks share device 0 (ATOS_SAME_DEVICE)")
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd, env=env)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=16)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="atos", choices=["atos", "reference"])
    ap.add_argument("--workload", default="bfs_rmat24", choices=sorted(WORKLOADS))
    ap.add_argument("--sources", type=int, default=16)
    ap.add_argument("--pr-steps", type=int, default=3)
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--no-pr", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--agg", type=int, default=1)
    ap.add_argument("--ctas-per-sm", type=int, default=0)
    ap.add_argument("--north-star", type=int, default=1, help="also time the RMAT-26 BFS target (N=1)")
    ap.add_argument("--extra-configs", type=int, default=1, help="also time configs[0], [3], [4] (N=1)")
    ap.add_argument("--c5", type=int, default=1, help="include configs[4] (PR RMAT-26, 8 virtual ranks)")
    ap.add_argument("--profile-range", action="store_true",
                    help="cudaProfilerStart/Stop around the timed region (ncu --profile-from-start off)")
    args = ap.parse_args()
    if args.warmup < 3:
        log("[bench] warmup raised to 3 (timing rule)")
        args.warmup = 3

    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn(args.gpus))
    rank, world, local = adist.init()
    if args.gpus > 1:
        assert world == args.gpus, f"--gpus {args.gpus} but WORLD_SIZE={world}"
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    assert torch.cuda.is_available(), "bench.py (impl atos) needs a CUDA device; no CPU fallback"
    same_dev = bool(os.environ.get("ATOS_SAME_DEVICE"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    from paper_conf_sc_chenbpbyo22_b200 import atos

    gname, app = WORKLOADS[args.workload]
    g = make_graph(gname, dev)
    deg = g.degrees()
    srcs = [0] if gname == "kron12" else inputs.bfs_sources(g, args.sources)
    stream = torch.cuda.current_stream(dev)
    cfg = dict(agg_enabled=args.agg, stream=stream.cuda_stream)
    if args.ctas_per_sm:
        cfg["ctas_per_sm"] = args.ctas_per_sm
    elif same_dev and world > 1:
        cfg["ctas_per_sm"] = 1            # time-sliced ranks on one device

    def load(rp, col, n, **kw):
        if world > 1:
            return adist.load_distributed(rp, col, n, **kw)
        return atos.Graph(rp, col, n, **kw)

    G = load(g.row_ptr, g.col, g.n, **cfg)
    depth = torch.empty(g.n, dtype=torch.int32, device=dev)

    # units per source (computed once from the device result; counting only)
    units = {}
    for s in srcs:
        G.bfs(s, depth_out=depth)
        G.sync()
        units[s] = m_reached_of(depth, deg)

    for k in range(args.warmup):
        G.bfs(srcs[k % len(srcs)], depth_out=depth)
        G.last_stats()

    seq = [srcs[(args.warmup + k) % len(srcs)] for k in range(args.steps)]
    worker_ms, edges_scanned, pops, hub_hits = [], 0, 0, 0
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(len(seq) + 1)]
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    if args.profile_range:
        torch.cuda.profiler.start()
    with ClockSampler(local) as clk:
        evs[0].record(stream)
        for i, s in enumerate(seq):
            G.bfs(s, depth_out=depth)
            st = G.last_stats()          # retires the solve (sync + error check), no extra device work
            evs[i + 1].record(stream)
            worker_ms.append(st["ms_worker"])
            edges_scanned += st["edges"]
            pops += st["pops"]
            hub_hits += st["hub_hits"]
        torch.cuda.synchronize()
    if args.profile_range:
        torch.cuda.profiler.stop()
    if world > 1:
        torch.distributed.barrier()
    step_ms = adist.max_over_ranks_vec([evs[i].elapsed_time(evs[i + 1]) for i in range(len(seq))])
    ms = adist.max_over_ranks(evs[0].elapsed_time(evs[-1]))
    m_total = sum(units[s][0] for s in seq)
    n_total = sum(units[s][1] for s in seq)
    value = m_total / (ms * 1e-3) / 1e9
    per_step = [units[s][0] / (t * 1e-3) / 1e9 for s, t in zip(seq, step_ms)]
    edges_scanned = int(adist.sum_over_ranks(edges_scanned))
    pops = int(adist.sum_over_ranks(pops))
    hub_hits = int(adist.sum_over_ranks(hub_hits))

    # roofline of the dominant kernel (the persistent worker), SURVEY §8d byte model
    peak, peak_src = peaks()
    bytes_per_launch = (8 * m_total + 28 * n_total) / len(seq) / world
    avg_worker_ms = adist.max_over_ranks(sum(worker_ms) / len(worker_ms))
    achieved = bytes_per_launch / (avg_worker_ms * 1e-3) / 1e9
    traffic = None
    prof = os.path.join(ROOT, "profiles", "ncu_worker_traffic.json")
    if os.path.exists(prof) and world == 1:
        try:
            pj = json.load(open(prof))
            if pj.get("workload") == args.workload:
                traffic = pj.get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": traffic, "kernel": "atos::worker_kernel<BFS>", "peak_source": peak_src,
            "bytes_model": "8*m_reached + 28*n_reached per BFS (SURVEY 8d), per rank",
            "worker_ms_avg": avg_worker_ms, "worker_share_of_step": avg_worker_ms / (ms / len(seq))}
    if world > 1:
        roof["multi_gpu"] = nvlink_roofline(g, deg, depth, G, seq[0], world, rank, peak, step_ms[0])

    cfgd = arm_config(args, g, srcs, world)
    if same_dev and world > 1:
        cfgd["same_device"] = "all ranks on device 0 (time-sliced): protocol check, not a scaling number"
    line = {"metric": METRIC,
            "value": value, "unit": "GTEPS", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms / len(seq), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic (seeded Graph500 RMAT, device-generated)",
            "config": cfgd,
            "gpu_launches": args.steps * (KERNELS_PER_BFS_STEP[1] + (1 if world > 1 else 0)),
            "roofline": roof,
            "per_source_gteps": {"harmonic_mean": statistics.harmonic_mean(per_step), "min": min(per_step),
                                 "max": max(per_step), "median_ms": statistics.median(step_ms),
                                 "mean_ms": statistics.mean(step_ms),
                                 "what": "one BFS per step from each of the sampled sources (Graph500 convention: "
                                         "harmonic mean); step times are max over ranks"},
            "counters": {"pops_per_reached": pops / max(1, n_total), "edges_per_m_reached": edges_scanned / max(1, m_total),
                         "hub_bound_retired_frac": hub_hits / max(1, edges_scanned)}}
    line["clocks"] = clk.summary()

    # ---- e2e: through the public API from pinned host memory, every step:
    # H2D of the CSR (graph_load), BFS, D2H of the depth array, free.
    rp_h = g.row_ptr.cpu().pin_memory()
    col_h = g.col.cpu().pin_memory()
    depth_h = torch.empty(g.n, dtype=torch.int32).pin_memory()
    if args.e2e_steps > 0:
        line["e2e"], line["e2e_query"] = e2e_block(args, G, load, cfg, rp_h, col_h, depth_h, g, seq, units, stream, world)

    # ---- PageRank line of the metric (configs[1])
    if not args.no_pr:
        line["pagerank"] = pagerank_block(args, dev, stream, cfg, load, world)

    # ---- CPU oracle baseline (rank 0, N = 1 only)
    if not args.no_cpu_baseline and world == 1 and rank == 0:
        s = seq[0]
        line["cpu_baseline"] = cpu_baseline_bfs(g, s, units[s][0])
        if not args.no_pr:
            line["cpu_baseline"]["pagerank_jacobi"] = cpu_baseline_pr()
    # ---- protocol overhead of the multi-rank path, measured with virtual ranks on this GPU
    if world == 1 and args.extra_configs and args.workload == "bfs_rmat24":
        line["virtual_ranks"] = virtual_rank_block(G_graph=g, srcs=seq, cfg=cfg, stream=stream, dev=dev)
    G.free()
    del g, deg, depth

    # ---- north_star target: BFS on RMAT-26 (symmetric) on one GPU
    if args.north_star and world == 1 and args.workload == "bfs_rmat24":
        torch.cuda.empty_cache()
        line["north_star_rmat26"] = north_star_block(dev, stream, cfg, peak)
    # ---- configs[0], configs[3], configs[4] (parity configs, reported beside the headline)
    if args.extra_configs and args.workload == "bfs_rmat24":
        torch.cuda.empty_cache()
        line["other_configs"] = other_configs(args, dev, stream, cfg, load, world)
    if rank == 0:
        print(json.dumps(line), flush=True)


def nvlink_roofline(g, deg, depth, G, src, world, rank, hbm_peak, step_ms):
    """Multi-GPU roofline: T_roof = max over ranks of max(B_HBM / HBM, B_NV / NVLink).
    B_NV = 8 B x M_out, M_out = distinct remote vertices adjacent to this rank's reached vertices
    (the minimum a push BFS with a sender-side filter must send), computed from the device depth."""
    G.bfs(src, depth_out=depth)
    G.sync()
    part = inputs.balanced_partition(g.n, world)
    lo, hi = part[rank], part[rank + 1]
    rp = g.row_ptr
    reached = depth[lo:hi] >= 0
    rows = torch.nonzero(reached).flatten() + lo
    m_r = int(deg[rows].sum())
    n_r = int(rows.numel())
    targets = []
    step = 1 << 22
    for a in range(0, rows.numel(), step):
        r = rows[a:a + step]
        cnt = (rp[r + 1] - rp[r])
        idx = torch.repeat_interleave(rp[r], cnt) + (torch.arange(int(cnt.sum()), device=rp.device) -
                                                      torch.repeat_interleave(torch.cumsum(cnt, 0) - cnt, cnt))
        v = g.col[idx].to(torch.int64)
        targets.append(torch.unique(v[(v < lo) | (v >= hi)]))
    m_out = int(torch.unique(torch.cat(targets)).numel()) if targets else 0
    b_hbm = 8 * m_r + 28 * n_r
    b_nv = 8 * m_out
    nv_peak = 770.0
    t_hbm = b_hbm / (hbm_peak * 1e9)
    t_nv = b_nv / (nv_peak * 1e9)
    t_roof = adist.max_over_ranks(max(t_hbm, t_nv))
    return {"bound": "nvlink" if adist.max_over_ranks(t_nv) > adist.max_over_ranks(t_hbm) else "hbm",
            "t_roof_ms": t_roof * 1e3, "t_step_ms": step_ms, "frac": t_roof * 1e3 / step_ms,
            "b_hbm_bytes_max_rank": adist.max_over_ranks(b_hbm), "b_nv_bytes_max_rank": adist.max_over_ranks(b_nv),
            "nvlink_peak_gbs": nv_peak, "nvlink_peak_source": "measured peer copy per direction (B200_PROFILING.md)",
            "source": src, "what": "B_NV = 8 B x distinct (rank, remote vertex) pairs reached via cut edges"}


def e2e_block(args, G, load, cfg, rp_h, col_h, depth_h, g, seq, units, stream, world):
    """load (pinned host CSR) + BFS (host depth out) + free per step, with a phase breakdown."""
    ecfg = dict(cfg, pool_retain=1)      # a load/solve/free loop keeps the pool's memory mapped
    H = load(rp_h, col_h, g.n, **ecfg)   # one untimed pass: first mapping of the pool
    H.bfs(seq[0], depth_out=depth_h)
    if world > 1:
        torch.distributed.barrier()
    H.free()
    e_units, ph = 0, {"load": [], "solve": [], "free": []}
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for k in range(args.e2e_steps):
        s = seq[k % len(seq)]
        t0 = time.perf_counter()
        H = load(rp_h, col_h, g.n, **ecfg)
        t1 = time.perf_counter()
        H.bfs(s, depth_out=depth_h)
        t2 = time.perf_counter()
        if world > 1:
            torch.distributed.barrier()     # peers may still read this rank's arena
        H.free()
        t3 = time.perf_counter()
        ph["load"].append((t1 - t0) * 1e3)
        ph["solve"].append((t2 - t1) * 1e3)
        ph["free"].append((t3 - t2) * 1e3)
        e_units += units[s][0]
    e1.record(stream)
    torch.cuda.synchronize()
    e_ms = adist.max_over_ranks(e0.elapsed_time(e1))
    e2e = {"value": e_units / (e_ms * 1e-3) / 1e9, "unit": "GTEPS",
           "h2d_bytes_per_step": int((g.n + 1) * 8 + g.nnz * 4),
           "d2h_bytes_per_step": int(g.n * 4), "steps": args.e2e_steps,
           "ms_per_step": e_ms / args.e2e_steps,
           "phase_ms_median": {k: statistics.median(v) for k, v in ph.items()},
           "phase_ms_max": {k: max(v) for k, v in ph.items()},
           "what": "atos_graph_load(pinned host CSR) + atos_bfs(host depth out) + atos_graph_free per step "
                   "(pool_retain=1: the freed graph's memory stays mapped for the next load)"}
    # query-only variant: graph resident, source in, host depth out
    torch.cuda.synchronize()
    q0, q1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    q0.record(stream)
    qu = 0
    for s in seq[:8]:
        G.bfs(s, depth_out=depth_h)
        qu += units[s][0]
    q1.record(stream)
    torch.cuda.synchronize()
    q_ms = adist.max_over_ranks(q0.elapsed_time(q1))
    q = {"value": qu / (q_ms * 1e-3) / 1e9, "unit": "GTEPS", "h2d_bytes_per_step": 8,
         "d2h_bytes_per_step": int(g.n * 4), "ms_per_step": q_ms / len(seq[:8]),
         "what": "graph resident; atos_bfs(src) -> pinned host depth"}
    return e2e, q


def pagerank_block(args, dev, stream, cfg, load, world):
    gp = make_graph("rmat20_pr", dev)
    # PR keeps the generator's (random) labels: degree relabeling measured 1.6x
    # slower for push-PR on RMAT-20
    P = load(gp.row_ptr, gp.col, gp.n, **dict(cfg, relabel=0))
    r_out = torch.empty(gp.n, dtype=torch.float64, device=dev)
    s_out = torch.empty(gp.n, dtype=torch.float64, device=dev)
    P.pagerank(0.85, 1e-9, rank_out=r_out, residual_out=s_out)
    P.last_stats()
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    relax, pr_pops, pr_worker, msgs = 0, 0, [], 0
    p0.record(stream)
    for _ in range(args.pr_steps):
        P.pagerank(0.85, 1e-9, rank_out=r_out, residual_out=s_out)
        st = P.last_stats()
        relax += st["edges"]
        pr_pops += st["pops"]
        msgs += st["msgs_sent"]
        pr_worker.append(st["ms_worker"])
    p1.record(stream)
    torch.cuda.synchronize()
    p_ms = adist.max_over_ranks(p0.elapsed_time(p1)) / args.pr_steps
    pr_worker_ms = adist.max_over_ranks(sum(pr_worker) / len(pr_worker))
    relax = adist.sum_over_ranks(relax) / args.pr_steps
    pr_pops = adist.sum_over_ranks(pr_pops) / args.pr_steps
    msgs = adist.sum_over_ranks(msgs) / args.pr_steps
    atom_peak = micro_peak("atomadd_f64_8MB_gops")
    if world > 1:
        torch.distributed.barrier()
    P.free()
    return {"workload": "pr_rmat20 (configs[1]) alpha=0.85 eps=1e-9", "graph": gp.name, "n_gpus": world,
            "n": gp.n, "nnz": gp.nnz, "ms_per_solve": p_ms,
            "gteps_relaxations": relax / (p_ms * 1e-3) / 1e9,
            "gteps_nnz_per_solve": gp.nnz / (p_ms * 1e-3) / 1e9,
            "relaxations_per_nnz": relax / gp.nnz, "pops_per_vertex": pr_pops / gp.n, "msgs_per_solve": msgs,
            "worker_ms_avg": pr_worker_ms, "dtype": "f64",
            "roofline": {"bound": "l2_atomic", "unit": "Gatomic/s",
                         "achieved": relax / world / (pr_worker_ms * 1e-3) / 1e9, "peak": atom_peak,
                         "frac": (relax / world / (pr_worker_ms * 1e-3) / 1e9 / atom_peak) if atom_peak else None,
                         "peak_source": "measured fp64 atomicAdd-with-return to random addresses "
                                        "in an 8 MB array (scripts/micro.cu, profiles/r1)"}}


def cpu_baseline_pr():
    """The oracle's Jacobi PageRank on configs[1] (RMAT-20 directed) on 1 core and on all cores."""
    import oracle
    import platform
    gp = inputs.make_config("rmat20_pr")
    rp, col = gp.numpy()
    out = {"graph": gp.name, "tol": 1e-12}
    # all cores: an explicit thread count (OMP_NUM_THREADS may be 1 in the environment;
    # the r2 box reported omp_get_max_threads() == 1 with 16 cores)
    ncores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
    for name, nt in (("one_core", 1), ("all_cores", ncores)):
        t0 = time.perf_counter()
        _, it, delta = oracle.pagerank(rp, col, 0.85, 1e-12, nthreads=nt)
        out[name] = {"seconds": time.perf_counter() - t0, "iterations": it, "threads": nt}
    out["nproc"] = os.cpu_count()
    try:
        out["cpu_model"] = next(l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name"))
    except Exception:
        out["cpu_model"] = platform.processor()
    return out


def virtual_rank_block(G_graph, srcs, cfg, stream, dev):
    """The multi-rank protocol's cost, measured on ONE GPU with virtual ranks (same SMs,
    channels in local HBM): BFS RMAT-24 and PR RMAT-20 at 1, 2 and 8 ranks."""
    from paper_conf_sc_chenbpbyo22_b200 import atos
    g = G_graph
    out = {"what": "same GPU, workers split among the ranks: protocol overhead, not scaling"}
    d = torch.empty(g.n, dtype=torch.int32, device=dev)
    deg = g.degrees().to(dev)
    pq = {"what": "N1 priority queue (Listing 4 threshold_delta, P:629-639) vs FIFO: redundant work as in "
                  "Table III (P:1333-1359) = edges scanned / m_reached and pops / reached, BFS RMAT-24, "
                  "virtual ranks on this GPU"}
    for vr in (1, 2, 8):
        for delta in (0, 1):
            H = atos.Graph(g.row_ptr, g.col, g.n, **dict(cfg, virtual_ranks=vr, pq_delta=delta))
            H.bfs(srcs[0], depth_out=d)
            H.last_stats()
            ws, ed, po = [], [], []
            for s in srcs[:4]:
                H.bfs(s, depth_out=d)
                st = H.last_stats()
                ws.append(st["ms_worker"])
                reached = d >= 0
                ed.append(st["edges"] / max(1, int(deg[reached].sum())))
                po.append(st["pops"] / max(1, int(reached.sum())))
            key = f"vr{vr}_" + ("fifo" if delta == 0 else f"pq{delta}")
            pq[key] = {"ms": statistics.median(ws), "edges_per_m_reached": statistics.mean(ed),
                       "pops_per_reached": statistics.mean(po)}
            if delta == 0:
                out[f"bfs_rmat24_vr{vr}_ms"] = statistics.median(ws)
                out[f"bfs_rmat24_vr{vr}_msgs_per_solve"] = st["msgs_sent"]
            H.free()
    out["priority_queue"] = pq
    gp = make_graph("rmat20_pr", dev)
    r_out = torch.empty(gp.n, dtype=torch.float64, device=dev)
    for vr in (1, 2, 8):
        H = atos.Graph(gp.row_ptr, gp.col, gp.n, **dict(cfg, relabel=0, virtual_ranks=vr))
        H.pagerank(0.85, 1e-9, rank_out=r_out)
        st = H.last_stats()
        out[f"pr_rmat20_vr{vr}_ms"] = st["ms_worker"]
        out[f"pr_rmat20_vr{vr}_msgs"] = st["msgs_sent"]
        H.free()
    return out


def north_star_block(dev, stream, cfg, peak):
    from paper_conf_sc_chenbpbyo22_b200 import atos
    g26 = make_graph("rmat26", dev)
    G26 = atos.Graph(g26.row_ptr, g26.col, g26.n, **cfg)
    d26 = torch.empty(g26.n, dtype=torch.int32, device=dev)
    deg26 = g26.degrees()
    srcs26 = inputs.bfs_sources(g26, 4)
    u26 = {}
    for s in srcs26:
        G26.bfs(s, depth_out=d26)
        G26.last_stats()
        u26[s] = m_reached_of(d26, deg26)
    torch.cuda.synchronize()
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(9)]
    wms, mt, nt, hh, ed = [], 0, 0, 0, 0
    evs[0].record(stream)
    for k in range(8):
        s = srcs26[k % len(srcs26)]
        G26.bfs(s, depth_out=d26)
        st = G26.last_stats()
        evs[k + 1].record(stream)
        wms.append(st["ms_worker"])
        hh += st["hub_hits"]
        ed += st["edges"]
        mt += u26[s][0]
        nt += u26[s][1]
    torch.cuda.synchronize()
    ms26 = evs[0].elapsed_time(evs[-1]) / 8
    steps = [evs[k].elapsed_time(evs[k + 1]) for k in range(8)]
    rates = [u26[srcs26[k % 4]][0] / (t * 1e-3) / 1e9 for k, t in enumerate(steps)]
    bytes26 = (8 * mt + 28 * nt) / 8
    w26 = sum(wms) / len(wms)
    G26.free()
    return {"workload": "bfs_rmat26 (north_star target: RMAT-26 ef16 symmetric BFS, 1 GPU)", "graph": g26.name,
            "n": g26.n, "nnz": g26.nnz, "gteps": mt / 8 / (ms26 * 1e-3) / 1e9, "ms_per_step": ms26,
            "gteps_harmonic_mean": statistics.harmonic_mean(rates), "gteps_min": min(rates), "gteps_max": max(rates),
            "hub_bound_retired_frac": hh / max(1, ed), "edges_per_m_reached": ed / max(1, mt),
            "roofline": {"bound": "hbm", "achieved": bytes26 / (w26 * 1e-3) / 1e9, "peak": peak, "unit": "GB/s",
                         "frac": bytes26 / (w26 * 1e-3) / 1e9 / peak, "bytes_model": "8*m_reached + 28*n_reached",
                         "worker_ms_avg": w26},
            "target": "frac >= 0.5 (BASELINE.json north_star)"}


def timed_bfs(G, src, depth, reps):
    """Device time (CUDA events on the launch stream) of `reps` BFS solves, ms each."""
    stream = torch.cuda.current_stream()
    G.bfs(src, depth_out=depth)
    st = G.last_stats()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    wms = []
    a.record(stream)
    for _ in range(reps):
        G.bfs(src, depth_out=depth)
        st = G.last_stats()
        wms.append(st["ms_worker"])
    b.record(stream)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps, sum(wms) / reps, st


def other_configs(args, dev, stream, cfg, load, world):
    from paper_conf_sc_chenbpbyo22_b200 import atos
    out = {}
    if world == 1:
        # configs[0]: Kronecker-12 from vertex 0 -- launch/latency bound (roofline meaningless, report us)
        g = make_graph("kron12", dev)
        G = atos.Graph(g.row_ptr, g.col, g.n, **cfg)
        d = torch.empty(g.n, dtype=torch.int32, device=dev)
        ms, wms, st = timed_bfs(G, 0, d, 20)
        m, nr = m_reached_of(d, g.degrees())
        out["kron12_bfs"] = {"workload": "configs[0] BFS from vertex 0, Kronecker-12 ef16", "n": g.n, "nnz": g.nnz,
                             "us_per_solve": ms * 1e3, "us_worker": wms * 1e3, "reached": nr,
                             "gteps": m / (ms * 1e-3) / 1e9, "bound": "launch/latency (0.8 MB graph)"}
        G.free()
        # latency floor: per-level time of the production kernel on a path graph
        npath = 100000
        idx = torch.arange(npath - 1, device=dev)
        gp = inputs.csr_from_edges(npath, idx, idx + 1, symmetrize=True, name="path1e5")
        G = atos.Graph(gp.row_ptr, gp.col, gp.n, **cfg)
        d = torch.empty(gp.n, dtype=torch.int32, device=dev)
        ms_path, wms_path, _ = timed_bfs(G, 0, d, 3)
        t_level_us = wms_path * 1e3 / npath
        G.free()
        # configs[3]: road-like grid from the corner (latency bound, ~11.8 K levels)
        g = make_graph("grid4900", dev)
        G = atos.Graph(g.row_ptr, g.col, g.n, **cfg)
        d = torch.empty(g.n, dtype=torch.int32, device=dev)
        ms, wms, st = timed_bfs(G, 0, d, 3)
        m, nr = m_reached_of(d, g.degrees())
        levels = int(d.max().item()) + 1
        t_lat = levels * t_level_us * 1e-3
        out["grid4900_bfs"] = {
            "workload": "configs[3] BFS from vertex 0 (corner), road-like grid 4900x4900", "n": g.n, "nnz": g.nnz,
            "ms_per_solve": ms, "ms_worker": wms, "gteps": m / (ms * 1e-3) / 1e9, "levels": levels,
            "us_per_level": wms * 1e3 / levels, "pops_per_reached": st["pops"] / nr,
            "edges_per_m_reached": st["edges"] / max(1, m),
            "roofline": {"bound": "latency", "unit": "ms", "achieved": wms, "peak": t_lat, "frac": t_lat / wms,
                         "what": "levels x per-level time of the same kernel on a 1e5-vertex path (the dependent "
                                 "pop->row->col->atomicMin->push chain), %.2f us/level" % t_level_us}}
        G.free()
        del g, d
        torch.cuda.empty_cache()
    # configs[4]: PageRank RMAT-26 directed, 8 ranks, aggregation on vs off.  One process per GPU when
    # the run has 8 (or N > 1) ranks; on one GPU the 8 ranks are virtual (one grid, same protocol,
    # channels in local HBM instead of over NVLink).
    if args.c5:
        g = make_graph("rmat26_pr", dev)
        r_out = torch.empty(g.n, dtype=torch.float64, device=dev)
        s_out = torch.empty(g.n, dtype=torch.float64, device=dev)
        ranks = "8 virtual ranks on 1 GPU: channels in local HBM, not NVLink" if world == 1 else \
            f"{world} processes, one per GPU (NVLink peer stores)" + (" -- time-sliced on one device" if
                                                                       os.environ.get("ATOS_SAME_DEVICE") else "")
        c5 = {"workload": f"configs[4] PageRank alpha=.85 eps=1e-9, RMAT-26 ef16 directed, {ranks}",
              "n": g.n, "nnz": g.nnz}
        # delta messages with aggregation on / off / N2 combining (the paper's comparison), and on
        # virtual ranks also the default there: remote atomics + activation messages for crossings
        modes = (("agg_on", 1, 0, 0), ("agg_off", 0, 0, 0), ("agg_on_combine_N2", 1, 1, 0))
        if world == 1:
            modes += (("remote_atomics_activations", 1, 0, 1),)
        for name, agg, comb, ratom in modes:
            extra = dict(relabel=0, agg_enabled=agg, pr_combine=comb)
            if world == 1:
                extra["virtual_ranks"] = 8
            if ratom:
                os.environ.pop("ATOS_PR_NORATOM", None)
            else:
                os.environ["ATOS_PR_NORATOM"] = "1"     # (read per solve by libatos)
            P = load(g.row_ptr, g.col, g.n, **dict(cfg, **extra))
            if world > 1:
                torch.distributed.barrier()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            P.pagerank(0.85, 1e-9, rank_out=r_out, residual_out=s_out)
            st = P.last_stats()
            b.record(stream)
            torch.cuda.synchronize()
            ms = adist.max_over_ranks(a.elapsed_time(b))
            wms = adist.max_over_ranks(st["ms_worker"])
            tot = {k: adist.sum_over_ranks(st[k]) for k in ("edges", "msgs_sent", "packets_sent", "bytes_sent")}
            bmax = adist.max_over_ranks(st["bytes_sent"])
            c5[name] = {
                "ms_per_solve": ms, "relaxations_per_nnz": tot["edges"] / g.nnz, "msgs": tot["msgs_sent"],
                "packets": tot["packets_sent"], "bytes_sent": tot["bytes_sent"],
                "msgs_per_packet": tot["msgs_sent"] / max(1, tot["packets_sent"]),
                "channel_GBps_total": tot["bytes_sent"] / (wms * 1e-3) / 1e9,
                "channel_GBps_max_rank": bmax / (wms * 1e-3) / 1e9,
                "nvlink_frac_max_rank": (bmax / (wms * 1e-3) / 1e9 / 770.0) if world > 1 else None,
                "gteps_relaxations": tot["edges"] / (ms * 1e-3) / 1e9}
            if world > 1:
                torch.distributed.barrier()
            P.free()
        os.environ.pop("ATOS_PR_NORATOM", None)
        out["rmat26_pr_8ranks" if world in (1, 8) else f"rmat26_pr_{world}ranks"] = c5
        del g, r_out, s_out
    return out


if __name__ == "__main__":
    main()

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
            "probe": "u8 depth-bound filter on skewed graphs (atos_config.probe_filter=auto)",
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=16)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="atos", choices=["atos", "reference"])
    ap.add_argument("--workload", default="bfs_rmat24", choices=sorted(WORKLOADS))
    ap.add_argument("--sources", type=int, default=16)
    ap.add_argument("--pr-steps", type=int, default=3)
    ap.add_argument("--e2e-steps", type=int, default=3)
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

    rank, world, local = adist.init()
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    assert torch.cuda.is_available(), "bench.py (impl atos) needs a CUDA device; no CPU fallback"
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
    if world > 1:
        G = adist.load_distributed(g.row_ptr, g.col, g.n, **cfg)
    else:
        G = atos.Graph(g.row_ptr, g.col, g.n, **cfg)
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
    worker_ms, edges_scanned, pops = [], 0, 0
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    if args.profile_range:
        torch.cuda.profiler.start()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for s in seq:
            G.bfs(s, depth_out=depth)
            st = G.last_stats()          # retires the solve (sync + error check), no extra device work
            worker_ms.append(st["ms_worker"])
            edges_scanned += st["edges"]
            pops += st["pops"]
        ev1.record(stream)
        torch.cuda.synchronize()
    if args.profile_range:
        torch.cuda.profiler.stop()
    if world > 1:
        torch.distributed.barrier()
    ms_rank = ev0.elapsed_time(ev1)
    ms = adist.max_over_ranks(ms_rank)
    m_total = sum(units[s][0] for s in seq)
    n_total = sum(units[s][1] for s in seq)
    value = m_total / (ms * 1e-3) / 1e9

    # roofline of the dominant kernel (the persistent worker), SURVEY §8d byte model
    peak, peak_src = peaks()
    bytes_per_launch = (8 * m_total + 28 * n_total) / len(seq) / world
    avg_worker_ms = adist.max_over_ranks(sum(worker_ms) / len(worker_ms))
    achieved = bytes_per_launch / (avg_worker_ms * 1e-3) / 1e9
    traffic = None
    prof = os.path.join(ROOT, "profiles", "ncu_worker_traffic.json")
    if os.path.exists(prof):
        try:
            pj = json.load(open(prof))
            if pj.get("workload") == args.workload:
                traffic = pj.get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": traffic, "kernel": "atos::worker_kernel<BFS>", "peak_source": peak_src,
            "bytes_model": "8*m_reached + 28*n_reached per BFS (SURVEY 8d)",
            "worker_ms_avg": avg_worker_ms, "worker_share_of_step": avg_worker_ms / (ms / len(seq))}
    chain_peak = micro_peak("chain_randseg_probe_occ2x512_gedges")
    scanned_rate = edges_scanned / len(seq) / world / (avg_worker_ms * 1e-3) / 1e9
    roof["l2_probe_view"] = {
        "what": "edges scanned per second vs the measured column-segment -> random-probe chain at the "
                "worker's occupancy (scripts/micro.cu): the binding hardware rate for this method",
        "achieved_gedges": scanned_rate, "peak_gedges": chain_peak,
        "frac": scanned_rate / chain_peak if chain_peak else None}

    line = {"metric": METRIC,
            "value": value, "unit": "GTEPS", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms / len(seq), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic (seeded Graph500 RMAT, device-generated)",
            "config": arm_config(args, g, srcs, world),
            "gpu_launches": args.steps * (KERNELS_PER_BFS_STEP[1] + (1 if world > 1 else 0)),
            "roofline": roof,
            "counters": {"pops_per_reached": pops / max(1, n_total), "edges_per_m_reached": edges_scanned / max(1, m_total)}}
    line["clocks"] = clk.summary()

    # ---- e2e: through the public API from pinned host memory, every step:
    # H2D of the CSR (graph_load), BFS, D2H of the depth array, free.
    rp_h = g.row_ptr.cpu().pin_memory()
    col_h = g.col.cpu().pin_memory()
    depth_h = torch.empty(g.n, dtype=torch.int32).pin_memory()
    if args.e2e_steps > 0:
        # one untimed pass first: the process's first multi-GB cudaMalloc maps memory
        # (~0.2 s once); the timed steps measure the steady state a serving loop sees
        H = atos.Graph(rp_h, col_h, g.n, **cfg) if world == 1 else adist.load_distributed(rp_h, col_h, g.n, **cfg)
        H.bfs(seq[0], depth_out=depth_h)
        H.free()
        e_units = 0
        if world > 1:
            torch.distributed.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for k in range(args.e2e_steps):
            s = seq[k % len(seq)]
            if world > 1:
                H = adist.load_distributed(rp_h, col_h, g.n, **cfg)
            else:
                H = atos.Graph(rp_h, col_h, g.n, **cfg)
            H.bfs(s, depth_out=depth_h)
            H.free()
            e_units += units[s][0]
        e1.record(stream)
        torch.cuda.synchronize()
        e_ms = adist.max_over_ranks(e0.elapsed_time(e1))
        line["e2e"] = {"value": e_units / (e_ms * 1e-3) / 1e9, "unit": "GTEPS",
                       "h2d_bytes_per_step": int((g.n + 1) * 8 + g.nnz * 4),
                       "d2h_bytes_per_step": int(g.n * 4), "steps": args.e2e_steps,
                       "what": "atos_graph_load(pinned host CSR) + atos_bfs(host depth out) + atos_graph_free per step"}
        # query-only variant: graph resident, source in, host depth out
        torch.cuda.synchronize()
        q0, q1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        q0.record(stream)
        qu = 0
        for s in seq[:4]:
            G.bfs(s, depth_out=depth_h)
            qu += units[s][0]
        q1.record(stream)
        torch.cuda.synchronize()
        q_ms = adist.max_over_ranks(q0.elapsed_time(q1))
        line["e2e_query"] = {"value": qu / (q_ms * 1e-3) / 1e9, "unit": "GTEPS", "h2d_bytes_per_step": 8,
                             "d2h_bytes_per_step": int(g.n * 4),
                             "what": "graph resident; atos_bfs(src) -> pinned host depth"}

    # ---- PageRank line of the metric (configs[1])
    if not args.no_pr and world == 1:
        gp = make_graph("rmat20_pr", dev)
        # PR keeps the generator's (random) labels: degree relabeling measured 1.6x
        # slower for push-PR on RMAT-20
        P = atos.Graph(gp.row_ptr, gp.col, gp.n, **dict(cfg, relabel=0))
        r_out = torch.empty(gp.n, dtype=torch.float64, device=dev)
        s_out = torch.empty(gp.n, dtype=torch.float64, device=dev)
        P.pagerank(0.85, 1e-9, rank_out=r_out, residual_out=s_out)
        P.last_stats()
        torch.cuda.synchronize()
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        relax, pr_pops, pr_worker = 0, 0, []
        p0.record(stream)
        for _ in range(args.pr_steps):
            P.pagerank(0.85, 1e-9, rank_out=r_out, residual_out=s_out)
            st = P.last_stats()
            relax += st["edges"]
            pr_pops += st["pops"]
            pr_worker.append(st["ms_worker"])
        p1.record(stream)
        torch.cuda.synchronize()
        p_ms = p0.elapsed_time(p1) / args.pr_steps
        pr_worker_ms = sum(pr_worker) / len(pr_worker)
        atom_peak = micro_peak("atomadd_f64_8MB_gops")
        line["pagerank"] = {"workload": "pr_rmat20 (configs[1]) alpha=0.85 eps=1e-9", "graph": gp.name,
                            "n": gp.n, "nnz": gp.nnz, "ms_per_solve": p_ms,
                            "gteps_relaxations": relax / args.pr_steps / (p_ms * 1e-3) / 1e9,
                            "gteps_nnz_per_solve": gp.nnz / (p_ms * 1e-3) / 1e9,
                            "relaxations_per_nnz": relax / args.pr_steps / gp.nnz,
                            "pops_per_vertex": pr_pops / args.pr_steps / gp.n,
                            "worker_ms_avg": pr_worker_ms, "dtype": "f64",
                            "roofline": {"bound": "l2_atomic", "unit": "Gatomic/s",
                                         "achieved": relax / args.pr_steps / (pr_worker_ms * 1e-3) / 1e9,
                                         "peak": atom_peak,
                                         "frac": (relax / args.pr_steps / (pr_worker_ms * 1e-3) / 1e9 / atom_peak)
                                         if atom_peak else None,
                                         "peak_source": "measured fp64 atomicAdd-with-return to random addresses "
                                                        "in an 8 MB array (scripts/micro.cu, profiles/r1)"}}
        P.free()

    # ---- CPU oracle baseline (rank 0, N = 1 only)
    if not args.no_cpu_baseline and world == 1 and rank == 0:
        s = seq[0]
        line["cpu_baseline"] = cpu_baseline_bfs(g, s, units[s][0])
    G.free()
    del g, deg, depth

    # ---- north_star target: BFS on RMAT-26 (symmetric) on one GPU
    if args.north_star and world == 1 and args.workload == "bfs_rmat24":
        torch.cuda.empty_cache()
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
        q0, q1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        wms, mt, nt = [], 0, 0
        q0.record(stream)
        for k in range(8):
            s = srcs26[k % len(srcs26)]
            G26.bfs(s, depth_out=d26)
            wms.append(G26.last_stats()["ms_worker"])
            mt += u26[s][0]
            nt += u26[s][1]
        q1.record(stream)
        torch.cuda.synchronize()
        ms26 = q0.elapsed_time(q1) / 8
        bytes26 = (8 * mt + 28 * nt) / 8
        w26 = sum(wms) / len(wms)
        line["north_star_rmat26"] = {
            "workload": "bfs_rmat26 (north_star target: RMAT-26 ef16 symmetric BFS, 1 GPU)", "graph": g26.name,
            "n": g26.n, "nnz": g26.nnz, "gteps": mt / 8 / (ms26 * 1e-3) / 1e9, "ms_per_step": ms26,
            "roofline": {"bound": "hbm", "achieved": bytes26 / (w26 * 1e-3) / 1e9, "peak": peak, "unit": "GB/s",
                         "frac": bytes26 / (w26 * 1e-3) / 1e9 / peak, "bytes_model": "8*m_reached + 28*n_reached"},
            "target": "frac >= 0.5 (BASELINE.json north_star)"}
        G26.free()
    # ---- configs[0], configs[3], configs[4] (parity configs, reported beside the headline)
    if args.extra_configs and world == 1 and args.workload == "bfs_rmat24":
        torch.cuda.empty_cache()
        line["other_configs"] = other_configs(args, dev, stream, cfg)
    if rank == 0:
        print(json.dumps(line), flush=True)


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


def other_configs(args, dev, stream, cfg):
    from paper_conf_sc_chenbpbyo22_b200 import atos
    out = {}
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
        "roofline": {"bound": "latency", "unit": "ms", "achieved": wms, "peak": t_lat, "frac": t_lat / wms,
                     "what": "levels x per-level time of the same kernel on a 1e5-vertex path (the dependent "
                             "pop->row->col->atomicMin->push chain), %.2f us/level" % t_level_us}}
    G.free()
    del g, d
    torch.cuda.empty_cache()
    # configs[4]: PageRank RMAT-26 directed, 8 ranks, aggregation on vs off.  One GPU in this run:
    # the 8 ranks are virtual (one grid, same protocol, channels in HBM instead of over NVLink).
    if args.c5:
        g = make_graph("rmat26_pr", dev)
        r_out = torch.empty(g.n, dtype=torch.float64, device=dev)
        s_out = torch.empty(g.n, dtype=torch.float64, device=dev)
        c5 = {"workload": "configs[4] PageRank alpha=.85 eps=1e-9, RMAT-26 ef16 directed, 8 ranks "
                          "(virtual ranks on 1 GPU: channels in local HBM, not NVLink)", "n": g.n, "nnz": g.nnz}
        for name, agg, comb in (("agg_on", 1, 0), ("agg_off", 0, 0), ("agg_on_combine_N2", 1, 1)):
            P = atos.Graph(g.row_ptr, g.col, g.n, **dict(cfg, relabel=0, virtual_ranks=8, agg_enabled=agg,
                                                         pr_combine=comb))
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            P.pagerank(0.85, 1e-9, rank_out=r_out, residual_out=s_out)
            st = P.last_stats()
            b.record(stream)
            torch.cuda.synchronize()
            ms = a.elapsed_time(b)
            c5[name] = {
                "ms_per_solve": ms, "relaxations_per_nnz": st["edges"] / g.nnz, "msgs": st["msgs_sent"],
                "packets": st["packets_sent"], "bytes_sent": st["bytes_sent"],
                "msgs_per_packet": st["msgs_sent"] / max(1, st["packets_sent"]),
                "channel_GBps": st["bytes_sent"] / (st["ms_worker"] * 1e-3) / 1e9,
                "gteps_relaxations": st["edges"] / (ms * 1e-3) / 1e9}
            P.free()
        out["rmat26_pr_8ranks"] = c5
        del g, r_out, s_out
    return out


if __name__ == "__main__":
    main()

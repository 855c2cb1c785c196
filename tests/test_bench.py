"""bench.py contract: --gpus N launches N ranks itself (torch.distributed.run, one
process per GPU) and the JSON line reports the whole job."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def last_json(out):
    for line in reversed(out.splitlines()):
        if line.startswith("{"):
            return json.loads(line)
    raise AssertionError(out[-3000:])


def test_reference_arm_spawns_ranks_and_only_rank0_prints():
    """CPU (gloo): --impl reference --gpus 2 re-launches itself with 2 ranks; rank 0 alone
    runs the oracle and prints one line; the other rank exits 0 without work."""
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                        "--workload", "bfs_kron12", "--steps", "2", "--warmup", "3"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["unit"] == "GTEPS" and d["value"] > 0


@pytest.mark.gpu
@pytest.mark.slow
def test_bench_gpus2_on_one_device():
    """bench.py --gpus 2 spawns 2 ranks (ATOS_SAME_DEVICE on a 1-GPU box) and
    reports n_gpus 2 with the multi-GPU roofline block."""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--workload", "bfs_rmat18",
                        "--steps", "3", "--warmup", "3", "--sources", "3", "--e2e-steps", "1", "--no-cpu-baseline",
                        "--north-star", "0", "--extra-configs", "0", "--pr-steps", "1"],
                       cwd=ROOT, capture_output=True, text=True, timeout=1200)
    assert r.returncode == 0, r.stderr[-4000:]
    d = last_json(r.stdout)
    assert d["n_gpus"] == 2 and d["value"] > 0
    assert d["roofline"]["multi_gpu"]["b_nv_bytes_max_rank"] > 0
    assert d["pagerank"]["n_gpus"] == 2

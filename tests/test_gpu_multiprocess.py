"""The real multi-process path -- IPC arena export/connect, the epoch barrier, the
coordinator's double wave and one-sided channel stores between processes -- with
two ranks time-sliced on the one GPU of the test box (scripts/mp_same_gpu.py)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_two_processes_same_gpu_bfs_and_pagerank():
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--standalone", "--nproc-per-node", "2",
           os.path.join(ROOT, "scripts", "mp_same_gpu.py")]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    out = r.stdout + r.stderr
    assert r.returncode == 0 and "MP_SAME_GPU PASS" in out, out[-4000:]


@pytest.mark.slow
@pytest.mark.parametrize("nproc", [3, 4])
def test_three_and_four_processes_same_gpu_rmat18(nproc):
    """The IPC / .sys path with 3 and 4 processes (time-sliced on one GPU) on RMAT-18."""
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", ATOS_MP_SCALE="18")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--standalone", "--nproc-per-node", str(nproc),
           os.path.join(ROOT, "scripts", "mp_same_gpu.py")]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    out = r.stdout + r.stderr
    assert r.returncode == 0 and "MP_SAME_GPU PASS" in out, out[-4000:]

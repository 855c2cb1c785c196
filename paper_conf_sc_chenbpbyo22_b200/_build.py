"""Build libatos.so (sm_100a SASS) in-tree with nvcc.  No GPU needed."""
from __future__ import annotations

import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.environ.get("ATOS_LIB") or os.path.join(PKG, "libatos.so")   # ATOS_LIB: experiment variants
SOURCES = [os.path.join(CSRC, "atos.cu")]
DEPS = SOURCES + [os.path.join(CSRC, f) for f in ("atos_rt.cuh", "atos_worker.cuh", "atos_aux.cuh", "atos_bfs1.cuh", "atos_qbench.cuh")] + \
    [os.path.join(ROOT, "include", "atos.h")]

NVCC_FLAGS = [
    "-O3", "-std=c++17",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-lineinfo",
    "-shared", "-Xcompiler", "-fPIC",
    "-cudart", "static",
    "-I", os.path.join(ROOT, "include"),
]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.sep not in c or os.path.exists(c)):
            return c
    return "nvcc"


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in DEPS if os.path.exists(d))


def variant() -> bool:
    """An experiment variant library was requested (ATOS_LIB)."""
    return bool(os.environ.get("ATOS_LIB"))


def source_commit() -> str:
    try:
        return subprocess.check_output(["git", "-C", ROOT, "rev-parse", "--short=12", "HEAD"],
                                       stderr=subprocess.DEVNULL, text=True).strip()
    except Exception:
        return "unknown"


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not stale():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    extra = os.environ.get("ATOS_NVCC_EXTRA", "").split()     # experiment variants (with ATOS_LIB)
    cmd = [nvcc()] + NVCC_FLAGS + extra + (["-Xptxas", "-v"] if verbose else []) + ["-o", tmp] + SOURCES
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    # provenance beside every built library (A/B variants must say what they are)
    dirty = ""
    try:
        if subprocess.check_output(["git", "-C", ROOT, "status", "--porcelain", "--", "paper_conf_sc_chenbpbyo22_b200/csrc",
                                    "include"], stderr=subprocess.DEVNULL, text=True).strip():
            dirty = " (sources modified after this commit)"
    except Exception:
        pass
    with open(LIB + ".info", "w") as f:
        f.write(f"commit {source_commit()}{dirty}\nATOS_NVCC_EXTRA={' '.join(extra)}\n")
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))

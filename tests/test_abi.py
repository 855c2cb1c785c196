"""C ABI: the library loads without a GPU, exports every symbol include/atos.h
declares, and its host-only entry points behave as documented."""
import ctypes
import os
import re

import numpy as np
import pytest
import torch

from paper_conf_sc_chenbpbyo22_b200 import atos

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    txt = open(os.path.join(ROOT, "include", "atos.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(atos_[a-z_]+)\s*\(", txt)))


def test_header_declares_expected_api():
    syms = declared_symbols()
    for s in ("atos_graph_load", "atos_bfs", "atos_pagerank", "atos_graph_free", "atos_last_error"):
        assert s in syms
    assert set(syms) == set(atos.EXPORTED)


def test_library_exports_every_declared_symbol():
    lib = atos.load()
    for s in declared_symbols():
        assert hasattr(lib, s), s


def test_struct_layouts_match_header():
    # field order/size of the ctypes mirror == C (checked through atos_config_init defaults)
    cfg = atos.default_config()
    assert cfg.worker_threads == 512 and cfg.fetch_size == 512
    assert cfg.n_ranks == 1 and cfg.virtual_ranks == 1 and cfg.stream is None
    # compile a probe against the header and compare every field offset
    import subprocess, tempfile
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "atos.h"', 'int main(void){']
    for cname, ct in (("atos_config", atos.Config), ("atos_stats", atos.Stats), ("atos_qbench_config", atos.QBenchConfig)):
        lines.append(f'printf("%zu\\n", sizeof({cname}));')
        for f, _ in ct._fields_:
            lines.append(f'printf("%zu\\n", offsetof({cname}, {f}));')
    lines.append("return 0;}")
    with tempfile.TemporaryDirectory() as d:
        src, exe = os.path.join(d, "p.c"), os.path.join(d, "p")
        open(src, "w").write("\n".join(lines))
        subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), src, "-o", exe])
        got = [int(x) for x in subprocess.check_output([exe]).split()]
    want = []
    for ct in (atos.Config, atos.Stats, atos.QBenchConfig):
        want.append(ctypes.sizeof(ct))
        want.extend(getattr(ct, f).offset for f, _ in ct._fields_)
    assert got == want


def test_version():
    assert atos.load().atos_version() == 5


def test_partition_balanced_matches_definition():
    for n, p in [(10, 3), (5, 8), (1 << 20, 8), (7, 1)]:
        assert atos.partition_balanced(n, p) == [(r * n) // p for r in range(p + 1)]
    with pytest.raises(atos.AtosError):
        atos.partition_balanced(10, 9)


def test_validate_csr():
    lib = atos.load()
    rp = np.array([0, 2, 3, 3], dtype=np.int64)
    col = np.array([1, 2, 0], dtype=np.int32)
    P = lambda a: a.ctypes.data_as(ctypes.c_void_p)
    assert lib.atos_validate_csr(P(rp), P(col), 3, 3) == 0
    bad = np.array([1, 5, 0], dtype=np.int32)
    assert lib.atos_validate_csr(P(rp), P(bad), 3, 3) == 1
    assert b"out of range" in lib.atos_last_error()
    rp2 = np.array([0, 2, 1, 3], dtype=np.int64)
    assert lib.atos_validate_csr(P(rp2), P(col), 3, 3) == 1


def test_arena_bytes_same_on_every_rank_shape():
    a = atos.arena_bytes(1 << 16, 4, 0, channel_packets=64)
    b = atos.arena_bytes(1 << 16, 4, 3, channel_packets=64)
    assert a == b and a > (1 << 16) * 12


def test_invalid_config_rejected_without_gpu():
    rp = np.array([0, 1, 1], dtype=np.int64)
    col = np.array([1], dtype=np.int32)
    with pytest.raises(atos.AtosError) as e:
        atos.Graph(rp, col, fetch_size=0)
    assert e.value.status == 1


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU failure mode")
def test_graph_load_fails_loudly_without_gpu():
    rp = np.array([0, 1, 1], dtype=np.int64)
    col = np.array([1], dtype=np.int32)
    with pytest.raises(atos.AtosError) as e:
        atos.Graph(rp, col)
    assert e.value.status == 2          # ATOS_ERR_CUDA: no silent CPU fallback


def test_relabel_and_hub_cache_config_validation():
    cfg = atos.default_config()
    assert cfg.relabel == 2 and cfg.hub_cache == -1          # auto / auto
    assert cfg.split_edges == -1 and cfg.keep_items == -1     # auto
    assert cfg.pq_delta == -1                                  # auto (N1 level buckets on large skewed graphs)
    rp = np.array([0, 1, 1], dtype=np.int64)
    col = np.array([1], dtype=np.int32)
    for bad in (dict(relabel=3), dict(hub_cache=33), dict(hub_cache=1 << 23), dict(hub_cache=-2),
                dict(hub_cache=32, virtual_ranks=2), dict(hub_cache=200), dict(split_edges=100), dict(split_edges=128),
                dict(split_edges=1 << 21), dict(split_edges=-2), dict(pr_combine=2), dict(keep_items=-2), dict(keep_mode=2), dict(discrete=2),
                dict(discrete=1, virtual_ranks=2), dict(discrete=1, n_ranks=2), dict(pq_delta=-2), dict(pq_threshold=-1)):
        with pytest.raises(atos.AtosError) as e:
            atos.Graph(rp, col, **bad)
        assert e.value.status == 1, bad


def test_queue_bench_rejects_bad_config_without_gpu():
    for kw in (dict(worker_size=16), dict(fetch_size=64, worker_size=32), dict(threads=1000), dict(rounds=0),
               dict(ring_cap=1000), dict(op="push", ring_cap=1024)):
        args = dict(worker_size=32, op="push_then_pop", threads=4096, rounds=10)
        args.update(kw)
        with pytest.raises((atos.AtosError, KeyError)) as e:
            atos.queue_bench(**args)
        if isinstance(e.value, atos.AtosError):
            assert e.value.status == 1, kw

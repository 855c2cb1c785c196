"""Seeded input generators: bit-reproducibility and structural properties."""
import numpy as np
import torch

from paper_conf_sc_chenbpbyo22_b200 import inputs


def _np_splitmix(key, counters):
    out = []
    with np.errstate(over="ignore"):
        for c in counters:
            z = np.uint64(key & (2 ** 64 - 1)) + np.uint64(c + 1) * np.uint64(0x9E3779B97F4A7C15)
            z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
            z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
            out.append(z ^ (z >> np.uint64(31)))
    return np.array(out, dtype=np.uint64)


def test_splitmix_matches_uint64_reference():
    key = inputs._key(7, 3)
    c = np.arange(0, 300, dtype=np.int64)
    got = inputs.splitmix64(key, torch.from_numpy(c)).numpy().view(np.uint64)
    assert np.array_equal(got, _np_splitmix(key, c.tolist()))


def test_label_bijection_is_permutation():
    for s in (1, 2, 5, 12, 13):
        x = torch.arange(1 << s, dtype=torch.int64)
        y = inputs._label_bijection(x, s, seed=9)
        assert torch.equal(torch.sort(y).values, x)


def _check_csr(g, symmetric):
    rp, col = g.numpy()
    assert rp[0] == 0 and rp[-1] == col.size and np.all(np.diff(rp) >= 0)
    assert col.min() >= 0 and col.max() < g.n
    src = np.repeat(np.arange(g.n), np.diff(rp))
    assert np.all(src != col)                               # no self-loops
    key = src.astype(np.int64) * g.n + col
    assert np.all(np.diff(key) > 0)                         # sorted, no duplicates
    if symmetric:
        rkey = np.sort(col.astype(np.int64) * g.n + src)
        assert np.array_equal(rkey, key)


def test_kron12_shape_and_determinism():
    g1 = inputs.make_config("kron12")
    g2 = inputs.make_config("kron12")
    assert torch.equal(g1.col, g2.col) and torch.equal(g1.row_ptr, g2.row_ptr)
    _check_csr(g1, True)
    deg = g1.degrees()
    assert 90_000 < g1.nnz < 105_000                        # ~64K generated, symmetrised, dedup'd
    assert int(deg[0]) == int(deg.max())                    # unpermuted: vertex 0 is the hub


def test_rmat_directed_and_permuted():
    g = inputs.rmat(11, 16, 1, symmetric=False)
    _check_csr(g, False)
    deg = g.degrees()
    assert int(deg.argmax()) != 0                           # permutation moved the hub
    assert float((deg == 0).float().mean()) > 0.2           # many dangling vertices


def test_grid_shape():
    g = inputs.road_grid(60, 40, seed=1)
    _check_csr(g, True)
    assert g.n == 2400
    avg = g.nnz / g.n
    assert 2.2 < avg < 2.8                                  # road_usa-like average degree


def test_sources_are_non_isolated_and_deterministic():
    g = inputs.rmat(10, 16, 1, symmetric=True)
    s1 = inputs.bfs_sources(g, 16)
    s2 = inputs.bfs_sources(g, 16)
    assert s1 == s2 and len(set(s1)) == 16
    deg = g.degrees()
    assert all(int(deg[s]) > 0 for s in s1)


def test_balanced_partition():
    assert inputs.balanced_partition(10, 3) == [0, 3, 6, 10]
    assert inputs.balanced_partition(5, 8)[-1] == 5

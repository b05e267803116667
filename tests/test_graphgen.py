"""Generator tests (host side): determinism, CSR well-formedness, hash reference."""
import numpy as np
import pytest
import torch

import graphgen as gg


def test_hash_matches_python_reference():
    idx = torch.tensor([0, 1, 2, 3, 1000, 123456789, 2 ** 40 + 7], dtype=torch.int64)
    for seed, stream in [(1, 0), (1, 1), (5, 1003), (2 ** 33 + 1, 7)]:
        got = gg.hash64(seed, stream, idx).tolist()
        ref = [gg._s64(gg.hash64_ref(seed, stream, int(i))) for i in idx]
        assert got == ref


def _well_formed(g):
    nindex, nlist = g.numpy()
    nindex = nindex.astype(np.int64)
    assert nindex[0] == 0 and nindex[-1] == len(nlist)
    assert np.all(np.diff(nindex) >= 0)
    assert len(nlist) == 0 or (nlist.min() >= 0 and nlist.max() < g.n)
    rows = np.repeat(np.arange(g.n), np.diff(nindex))
    assert not np.any(rows == nlist), "self-loop"
    key = rows.astype(np.int64) * g.n + nlist
    assert np.all(np.diff(key) > 0), "rows must be sorted and deduplicated"
    rkey = nlist.astype(np.int64) * g.n + rows
    assert np.array_equal(np.sort(rkey), key), "graph must be symmetric"


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_configs_small_well_formed_and_deterministic(name):
    sd = {"C1": 4, "C2": 8, "C3": 10, "C4": 12, "C5": 15}[name]
    g1 = gg.make_config(name, seed=2, scale_down=sd)
    g2 = gg.make_config(name, seed=2, scale_down=sd)
    _well_formed(g1)
    assert torch.equal(g1.nindex, g2.nindex) and torch.equal(g1.nlist, g2.nlist)
    g3 = gg.make_config(name, seed=3, scale_down=sd)
    assert not (g1.m == g3.m and torch.equal(g1.nlist, g3.nlist))


def test_bucketed_csr_equals_single_sort():
    g1 = gg.rmat(12, 8, seed=4, buckets=1)
    g2 = gg.rmat(12, 8, seed=4, buckets=5)
    assert torch.equal(g1.nindex, g2.nindex) and torch.equal(g1.nlist, g2.nlist)


def test_permutation_is_bijection():
    p = gg.vertex_permutation(1000, seed=9)
    assert torch.equal(torch.sort(p).values, torch.arange(1000))


def test_shuffle_rows_keeps_row_sets():
    g = gg.erdos_renyi(300, 900, seed=3)
    s = gg.shuffle_rows(g, seed=1)
    nindex = g.nindex.tolist()
    changed = False
    for v in range(g.n):
        a = g.nlist[nindex[v]:nindex[v + 1]].tolist()
        b = s.nlist[nindex[v]:nindex[v + 1]].tolist()
        assert sorted(a) == sorted(b)
        changed |= a != b
    assert changed


def test_grid_deletion_rate():
    g = gg.grid2d(256, 256, 0.10, seed=1)
    full = 2 * 2 * 256 * 255
    assert abs(g.m / full - 0.9) < 0.01


def test_inject_loops_dups_raw_csr():
    """The raw-CSR generator keeps every original entry, adds loops and (symmetric)
    duplicates, and leaves the components unchanged (oracle O1 on both)."""
    import oracle
    g = gg.make_config("C1", seed=2, scale_down=4)
    r = gg.inject_loops_dups(g, seed=3, p_loop=0.2, p_dup=0.2)
    ni, nl = r.numpy()
    ni = ni.astype(np.int64)
    assert ni[0] == 0 and ni[-1] == len(nl) and np.all(np.diff(ni) >= 0)
    rows = np.repeat(np.arange(r.n), np.diff(ni))
    assert np.any(rows == nl), "no self-loop injected"
    key = rows.astype(np.int64) * r.n + nl
    assert len(np.unique(key)) < len(key), "no duplicate injected"
    assert np.any(np.diff(key) < 0), "rows not shuffled"
    # same multiset of distinct non-loop entries as the clean graph, and symmetric
    clean = np.unique(key[rows != nl])
    g_ni, g_nl = g.numpy()
    g_rows = np.repeat(np.arange(g.n), np.diff(g_ni.astype(np.int64)))
    assert np.array_equal(clean, g_rows.astype(np.int64) * g.n + g_nl)
    rkey = nl.astype(np.int64) * r.n + rows
    assert np.array_equal(np.sort(rkey), np.sort(key))
    assert np.array_equal(oracle.bfs(ni, nl)[0], oracle.bfs(*g.numpy())[0])

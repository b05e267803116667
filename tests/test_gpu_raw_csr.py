"""GPU parity on RAW CSRs: self-loops, duplicate entries and unsorted rows (SURVEY §8(b)
"accepted inputs", §8(c) pin "self-loops + duplicates -> same as cleaned"; DESIGN R8).

The graphs here are assembled entry by entry (``graphgen.raw_csr``) or by injecting loops
and duplicates into a config graph (``graphgen.inject_loops_dups``) — never through
``csr_from_pairs``, which cleans them away.  The expected labels are oracle O1 on
the same uncleaned CSR, and they must also equal O1 on the cleaned graph.  Covered entry
points: ecl_cc_run (int32 offsets), ecl_cc_run_i64, ecl_cc_spanning_forest; kernel orders
0 (the paper's) and 2 (concurrent, the default).
"""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle
import paper_conf_hpdc_jaiganeshb18_b200 as ecl

pytestmark = pytest.mark.gpu

SMALL = {"C1": 0, "C2": 4, "C3": 4, "C4": 6, "C5": 10}


@pytest.fixture(scope="module")
def h():
    with ecl.Handle(0) as handle:
        yield handle


def rows_graph(name, n, rows, seed=None):
    """Raw CSR from {v: [entries in row order]} (directed entries, as listed)."""
    R, C = [], []
    for v in sorted(rows):
        R += [v] * len(rows[v])
        C += list(rows[v])
    return gg.raw_csr(name, n, torch.tensor(R, dtype=torch.int64),
                      torch.tensor(C, dtype=torch.int64), seed=seed)


def undirected_raw(name, n, pairs, loops=(), seed=None):
    """Both directions of every listed pair (repeats kept) plus the listed loops."""
    R = [a for a, b in pairs] + [b for a, b in pairs] + list(loops)
    C = [b for a, b in pairs] + [a for a, b in pairs] + list(loops)
    return gg.raw_csr(name, n, torch.tensor(R, dtype=torch.int64),
                      torch.tensor(C, dtype=torch.int64), seed=seed)


def hand_raw_graphs():
    G = []
    # loops and a doubled edge: {0}, {1, 2, 3}
    G.append(rows_graph("loops_doubled", 4, {0: [0, 0], 1: [1, 2, 2, 1], 2: [1, 1, 2, 3],
                                             3: [2, 3, 3]}))
    # only loops: every vertex its own component
    G.append(rows_graph("only_loops", 5, {v: [v] * (v + 1) for v in range(5)}))
    # Init3 parent duplicated ahead of another smaller neighbour (R24's "other" test): row 5
    # = [3, 3, 1, 7] has hook work on (5, 1); row 6 = [4, 4, 8, 6] has none beyond its parent
    G.append(rows_graph("dup_parent_first", 9, {
        1: [5], 3: [5, 5], 4: [6, 6], 5: [3, 3, 1, 7], 6: [4, 4, 8, 6], 7: [5], 8: [6]}))
    # a vertex whose row is one neighbour repeated, at every bin size (P:L155 thresholds)
    pairs, base = [], 0
    for d in (3, 16, 17, 352, 353, 2000):
        pairs += [(base + 1, base)] * d          # (v, u) with v > u repeated d times
        pairs += [(base + 1, base + 1)]          # and a loop pair on the same row
        base += 2
    G.append(undirected_raw("repeated_single_neighbour", base, pairs))
    # hubs of every bin with a loop first in the row and every leaf edge doubled
    pairs, loops, base = [], [], 0
    for d in (15, 16, 17, 351, 352, 353, 1000):
        hub = base + d                           # largest ID: active, hooks all leaves
        loops += [hub, hub]
        pairs += [(hub, base + i) for i in range(d)] * 2
        base += d + 1
    G.append(undirected_raw("hubs_loops_doubled", base, pairs, loops, seed=7))
    # a long reversed chain whose every edge appears three times, loops on every 3rd vertex
    n = 50_000
    pairs = [(v, v - 1) for v in range(1, n)] * 3
    G.append(undirected_raw("chain_x3", n, pairs, loops=range(0, n, 3), seed=3))
    return G


def labels(h, g, index_dtype=None, **opts):
    g = g.to("cuda")
    nindex = g.nindex if index_dtype is None else g.nindex.to(index_dtype)
    for k, v in opts.items():
        h.set_option(k, v)
    try:
        out = h.run(nindex, g.nlist)
        torch.cuda.synchronize()
    finally:
        h.set_option("order", 2)
        h.set_option("prejump", 2)
        h.set_option("fuse_init", 2)
    return out.cpu().numpy()


def expected(g):
    nidx, nl = g.numpy()
    lab, ncc = oracle.bfs(nidx, nl)
    assert oracle.check(nidx, nl, lab, ncc) == 0
    return lab


def has_loops_and_dups(g):
    ni, nl = g.numpy()
    rows = np.repeat(np.arange(g.n), np.diff(ni.astype(np.int64)))
    key = rows.astype(np.int64) * g.n + nl
    return bool(np.any(rows == nl)), len(np.unique(key)) < len(key)


@pytest.mark.parametrize("g", hand_raw_graphs(), ids=lambda g: g.name)
@pytest.mark.parametrize("order", [0, 2])
@pytest.mark.parametrize("index_dtype", [torch.int32, torch.int64], ids=["i32", "i64"])
@pytest.mark.parametrize("fuse", [0, 1, 2])
def test_hand_raw(h, g, order, index_dtype, fuse):
    exp = expected(g)
    got = labels(h, g, index_dtype=index_dtype, order=order, fuse_init=fuse)
    assert np.array_equal(got, exp), g.name


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("order", [0, 2])
def test_configs_with_loops_dups(h, name, order):
    clean = gg.make_config(name, seed=31, scale_down=SMALL[name], device="cuda")
    g = gg.inject_loops_dups(clean, seed=5)
    assert has_loops_and_dups(g) == (True, True)
    exp = expected(g)
    assert np.array_equal(exp, expected(clean))          # "same as cleaned"
    assert np.array_equal(labels(h, g, order=order), exp)
    assert np.array_equal(labels(h, g, index_dtype=torch.int64, order=order), exp)
    for fuse in (0, 1, 2):
        assert np.array_equal(labels(h, g, order=order, fuse_init=fuse), exp)


@pytest.mark.parametrize("name", ["C4", "C5"])
@pytest.mark.parametrize("opts", [dict(filter=1), dict(prejump=1), dict(load_mode=0)],
                         ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
def test_configs_with_loops_dups_options(h, name, opts):
    clean = gg.make_config(name, seed=32, scale_down=SMALL[name] - 1, device="cuda")
    g = gg.inject_loops_dups(clean, seed=6, p_loop=0.3, p_dup=0.3)
    try:
        assert np.array_equal(labels(h, g, **opts), expected(g))
    finally:
        h.set_option("filter", 2)
        h.set_option("load_mode", 1)


@pytest.mark.parametrize("g", hand_raw_graphs()[:5], ids=lambda g: g.name)
def test_hand_raw_init_stage(h, g):
    """Init3 on raw rows: the first entry in row order that is smaller than v."""
    got = labels(h, g, stop_after=1)
    h.set_option("stop_after", 0)
    assert np.array_equal(got, oracle.init3(*g.numpy()))


def _forest(h, g, index_dtype=None, order=2, fuse=2):
    g = g.to("cuda")
    nindex = g.nindex if index_dtype is None else g.nindex.to(index_dtype)
    h.set_option("order", order).set_option("fuse_init", fuse)
    try:
        lab, ta, tb = h.spanning_forest(nindex, g.nlist)
        torch.cuda.synchronize()
    finally:
        h.set_option("order", 2).set_option("fuse_init", 2)
    nidx, nl = g.numpy()
    exp = expected(g)
    assert np.array_equal(lab.cpu().numpy(), exp)
    ta, tb = ta.cpu().numpy(), tb.cpu().numpy()
    assert oracle.check_forest(nidx, nl, exp, ta, tb) == 0
    m = ta >= 0
    assert not np.any(ta[m] == tb[m]), "a self-loop became a tree edge"


@pytest.mark.parametrize("g", hand_raw_graphs(), ids=lambda g: g.name)
@pytest.mark.parametrize("order", [0, 2])
@pytest.mark.parametrize("fuse", [0, 1, 2])
def test_forest_hand_raw(h, g, order, fuse):
    _forest(h, g, order=order, fuse=fuse)


@pytest.mark.parametrize("name", ["C2", "C4", "C5"])
def test_forest_configs_with_loops_dups(h, name):
    g = gg.inject_loops_dups(gg.make_config(name, seed=33, scale_down=SMALL[name],
                                            device="cuda"), seed=8)
    _forest(h, g, order=0)
    _forest(h, g, index_dtype=torch.int64, order=2)
    _forest(h, g, order=2, fuse=1)

"""Pins for the CPU oracle (oracle/), independent of the oracle's own code.

Each pin is something other than the oracle itself: exhaustive brute force by transitive
closure, scipy's connected_components, hand-built graphs whose answers are worked out by
hand, the paper's printed values (Table 2, Fig. 2 prose), and mutation tests showing the
invariant checker rejects each plausible wrong labelling.
"""
import itertools
import json
import os

import numpy as np
import pytest

import graphgen as gg
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def csr_np(n, edges):
    """Plain numpy CSR from undirected edges; keeps duplicates/self-loops as given."""
    rows = [[] for _ in range(n)]
    for a, b in edges:
        rows[a].append(b)
        if a != b:
            rows[b].append(a)
        else:
            rows[a].append(a)
    nindex = np.zeros(n + 1, dtype=np.int64)
    for v in range(n):
        nindex[v + 1] = nindex[v] + len(rows[v])
    nlist = np.array([u for r in rows for u in r], dtype=np.int32)
    return nindex, nlist


def closure_labels(adj):
    """Brute force: boolean transitive closure by repeated squaring (Warshall-style), then
    label[v] = smallest w reachable from v.  adj: (G, n, n) bool."""
    G, n, _ = adj.shape
    R = adj | np.eye(n, dtype=bool)[None]
    for _ in range(max(1, int(np.ceil(np.log2(max(n, 2)))) + 1)):
        R = (R.astype(np.int32) @ R.astype(np.int32)) > 0
    return np.argmax(R, axis=2).astype(np.int32)  # first True = min reachable ID


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 6])
def test_exhaustive_all_graphs(n):
    pairs = list(itertools.combinations(range(n), 2))
    G = 1 << len(pairs)
    adj = np.zeros((G, n, n), dtype=bool)
    for k, (a, b) in enumerate(pairs):
        on = ((np.arange(G) >> k) & 1).astype(bool)
        adj[:, a, b] = on
        adj[:, b, a] = on
    expect = closure_labels(adj)
    for g in range(G):
        edges = [pairs[k] for k in range(len(pairs)) if (g >> k) & 1]
        nindex, nlist = csr_np(n, edges)
        lb, ncc_b = oracle.bfs(nindex, nlist)
        lu, ncc_u = oracle.uf(nindex, nlist)
        assert np.array_equal(lb, expect[g]), (n, edges)
        assert np.array_equal(lu, expect[g]), (n, edges)
        assert ncc_b == ncc_u == len(set(expect[g].tolist()))
        assert oracle.check(nindex, nlist, lb, ncc_b) == 0


def test_scipy_random_graphs():
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import connected_components
    rng = np.random.default_rng(12345)
    for trial in range(300):
        n = int(rng.integers(1, 2000))
        m = int(rng.integers(0, 3 * n))
        a = rng.integers(0, n, m)
        b = rng.integers(0, n, m)
        nindex, nlist = csr_np(n, zip(a.tolist(), b.tolist()))
        A = csr_matrix((np.ones(len(nlist)), nlist, nindex), shape=(n, n))
        ncc, comp = connected_components(A, directed=False)
        cmin = np.full(ncc, n, dtype=np.int64)
        np.minimum.at(cmin, comp, np.arange(n))
        expect = cmin[comp].astype(np.int32)
        lb, nb = oracle.bfs(nindex, nlist)
        lu, nu = oracle.uf(nindex, nlist)
        assert nb == nu == ncc
        assert np.array_equal(lb, expect)
        assert np.array_equal(lu, expect)
        assert oracle.check(nindex, nlist, lb, ncc) == 0


def _both(n, edges):
    nindex, nlist = csr_np(n, edges)
    lb, nb = oracle.bfs(nindex, nlist)
    lu, nu = oracle.uf(nindex, nlist)
    assert np.array_equal(lb, lu) and nb == nu
    assert oracle.check(nindex, nlist, lb, nb) == 0
    return lb.tolist(), nb


def test_hand_built_graphs():
    assert _both(0, []) == ([], 0)
    assert _both(1, []) == ([0], 1)
    assert _both(5, []) == ([0, 1, 2, 3, 4], 5)
    # a path visiting the IDs in a scrambled order: 4-2-0-3-1 -> one component, min 0
    assert _both(5, [(4, 2), (2, 0), (0, 3), (3, 1)]) == ([0] * 5, 1)
    # path whose minimum sits at one end and whose IDs descend: 5-4-3-2-1 plus isolated 0
    assert _both(6, [(5, 4), (4, 3), (3, 2), (2, 1)]) == ([0, 1, 1, 1, 1, 1], 2)
    # two interleaved cliques on evens / odds
    ev = [(a, b) for a in range(0, 10, 2) for b in range(a + 2, 10, 2)]
    od = [(a, b) for a in range(1, 10, 2) for b in range(a + 2, 10, 2)]
    assert _both(10, ev + od) == ([0, 1] * 5, 2)
    # star with centre n-1 (every leaf is an Init3 root) and star with centre 0
    assert _both(500, [(499, i) for i in range(499)]) == ([0] * 500, 1)
    assert _both(500, [(0, i) for i in range(1, 400)]) == ([0] * 400 + list(range(400, 500)), 101)
    # K_40 clique
    assert _both(40, list(itertools.combinations(range(40), 2))) == ([0] * 40, 1)
    # self-loops and duplicate edges change nothing
    assert _both(4, [(1, 1), (2, 3), (3, 2), (2, 3), (0, 0)]) == ([0, 1, 2, 2], 3)


def test_fig2_prose_example():
    """Fig. 2 prose: hooking edge (6,8) with reps 3 and 7 points 7 at 3."""
    lines = [ln.split() for ln in open(os.path.join(GOLDEN, "fig2_hook.txt"))
             if ln.strip() and not ln.startswith("#")]
    n = int(lines[0][0])
    edges = [(int(a), int(b)) for a, b in lines[1:-1]]
    expect = [int(x) for x in lines[-1]]
    labels, ncc = _both(n, edges)
    assert labels == expect and ncc == 7


def test_long_reversed_chain():
    """Each v adjacent to v-1 (n = 2^20): worst-case pointer chains, one component."""
    n = 1 << 20
    g = gg.from_edges(n, [(v, v - 1) for v in range(n - 1, 0, -1)])
    lb, nb = oracle.bfs(*g.numpy())
    lu, nu = oracle.uf(*g.numpy())
    assert nb == nu == 1 and not lb.any() and not lu.any()


def test_init3_by_hand():
    """Init3: first neighbour *in adjacency order* with a smaller ID, else self."""
    nindex = np.array([0, 1, 3, 3, 6, 8], dtype=np.int64)
    #          v=0: [3]   v=1: [4, 0]  v=2: []  v=3: [4, 2, 0]  v=4: [1, 3]
    nlist = np.array([3, 4, 0, 4, 2, 0, 1, 3], dtype=np.int32)
    assert oracle.init3(nindex, nlist).tolist() == [0, 0, 2, 2, 1]
    # not the minimum neighbour (that would be Init2): v=3 takes 2, not 0
    nlist2 = np.array([3, 4, 0, 0, 2, 4, 3, 1], dtype=np.int32)
    assert oracle.init3(nindex, nlist2).tolist() == [0, 0, 2, 0, 3]


def test_check_rejects_wrong_labellings():
    # two components {0,1,2} and {3,4}, isolated 5
    nindex, nlist = csr_np(6, [(0, 1), (1, 2), (3, 4)])
    good = np.array([0, 0, 0, 3, 3, 5], dtype=np.int32)
    assert oracle.check(nindex, nlist, good, 3) == 0
    split = np.array([0, 0, 2, 3, 3, 5], dtype=np.int32)      # component split: I1
    assert oracle.check(nindex, nlist, split, 3) == 1
    maxid = np.array([2, 2, 2, 4, 4, 5], dtype=np.int32)      # max-ID convention: I2
    assert oracle.check(nindex, nlist, maxid, 3) == 2
    notself = np.array([0, 0, 0, 0, 0, 5], dtype=np.int32)     # label not a root... merged: I3
    assert oracle.check(nindex, nlist, notself, 3) == 3
    chain = np.array([0, 0, 0, 1, 1, 5], dtype=np.int32)       # label[label[v]] != label[v]? 1->0
    assert oracle.check(nindex, nlist, chain, 3) == 2
    oob = np.array([0, 0, 0, 3, 3, 6], dtype=np.int32)
    assert oracle.check(nindex, nlist, oob, 3) == 4


def test_table2_grid_exact():
    """2d-2e20.sym row of Table 2: n, m, dmin, davg, dmax, #CC all exact."""
    row = json.load(open(os.path.join(GOLDEN, "table2.json")))["2d-2e20.sym"]
    g = gg.grid2d(1024, 1024, 0.0)
    d = g.degrees()
    assert (g.n, g.m) == (row["n"], row["m"])
    assert (int(d.min()), int(d.max())) == (row["dmin"], row["dmax"])
    assert round(float(d.double().mean()), 1) == row["davg"]
    labels, ncc = oracle.bfs(*g.numpy())
    assert ncc == row["ccs"] and not labels.any()
    lu, nu = oracle.uf(*g.numpy())
    assert nu == 1 and not lu.any()


def test_table2_rmat16_statistical():
    row = json.load(open(os.path.join(GOLDEN, "table2.json")))["rmat16.sym"]
    g = gg.rmat(16, 8, (0.55, 0.10, 0.10), seed=1)
    d = g.degrees()
    _, ncc = oracle.bfs(*g.numpy())
    assert g.n == row["n"]
    assert abs(g.m - row["m"]) / row["m"] < 0.01
    assert abs(int(d.max()) - row["dmax"]) / row["dmax"] < 0.15
    assert abs(ncc - row["ccs"]) / row["ccs"] < 0.15
    _, nu = oracle.uf(*g.numpy())
    assert nu == ncc


def test_table2_r4_statistical_small():
    """r4 recipe at 2^20 vertices: 4-out random graphs are connected (Table 2 r4-2e23: 1 CC)."""
    g = gg.random_kout(1 << 20, 4, seed=1)
    d = g.degrees()
    _, ncc = oracle.bfs(*g.numpy())
    assert ncc == 1
    assert int(d.min()) >= 4 and abs(float(d.double().mean()) - 8.0) < 0.01


# ---- spanning-forest checker (oracle_check_forest) ----------------------

def _slots(n, labels, edges, rng):
    """Assign a list of undirected edges to the non-minimum vertices' slots (the CUDA
    path's output format), each edge in a random orientation; minima get (-1, -1)."""
    ta = np.full(n, -1, dtype=np.int32)
    tb = np.full(n, -1, dtype=np.int32)
    slots = [x for x in range(n) if labels[x] != x]
    assert len(slots) == len(edges)
    for x, (a, b) in zip(slots, edges):
        if rng.random() < 0.5:
            a, b = b, a
        ta[x], tb[x] = a, b
    return ta, tb


def _closure_classes(n, edges):
    adj = np.zeros((1, n, n), dtype=bool)
    for a, b in edges:
        adj[0, a, b] = adj[0, b, a] = True
    return len(set(closure_labels(adj)[0].tolist()))


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5])
def test_forest_checker_brute_force(n):
    """Every subset S of a graph's edges with |S| = n - #CC is fed to the checker; it must
    accept exactly the subsets whose transitive closure has #CC classes (brute force)."""
    rng = np.random.default_rng(n)
    pairs = list(itertools.combinations(range(n), 2))
    graphs = range(1 << len(pairs))
    if n == 5:
        graphs = rng.choice(1 << len(pairs), 150, replace=False)
    for g in graphs:
        edges = [pairs[k] for k in range(len(pairs)) if (int(g) >> k) & 1]
        nindex, nlist = csr_np(n, edges)
        labels, ncc = oracle.bfs(nindex, nlist)
        for S in itertools.combinations(edges, n - ncc):
            ta, tb = _slots(n, labels, list(S), rng)
            spans = _closure_classes(n, S) == ncc
            rc = oracle.check_forest(nindex, nlist, labels, ta, tb)
            assert rc == (0 if spans else 3), (n, edges, S, rc)


def test_forest_checker_mutations():
    g = gg.erdos_renyi(3000, 4000, seed=5)
    nindex, nlist = g.numpy()
    labels, ncc = oracle.bfs(nindex, nlist)
    ta, tb, ncc2 = oracle.bfs_forest(nindex, nlist)
    assert ncc2 == ncc
    assert oracle.check_forest(nindex, nlist, labels, ta, tb) == 0
    non_min = np.flatnonzero(labels != np.arange(g.n))
    x = int(non_min[7])
    # a pair that is not a CSR entry
    a, b = ta.copy(), tb.copy()
    row = set(nlist[nindex[a[x]]:nindex[a[x] + 1]].tolist())
    b[x] = next(w for w in range(g.n) if w not in row and w != a[x])
    assert oracle.check_forest(nindex, nlist, labels, a, b) == 2
    # out of range
    a, b = ta.copy(), tb.copy()
    b[x] = g.n
    assert oracle.check_forest(nindex, nlist, labels, a, b) == 2
    # a non-minimum slot left empty / a minimum slot filled
    a, b = ta.copy(), tb.copy()
    a[x] = b[x] = -1
    assert oracle.check_forest(nindex, nlist, labels, a, b) == 1
    a, b = ta.copy(), tb.copy()
    mn = int(np.flatnonzero(labels == np.arange(g.n))[0])
    a[mn], b[mn] = ta[x], tb[x]
    assert oracle.check_forest(nindex, nlist, labels, a, b) == 1
    # a duplicated tree edge: some slot repeats another slot's edge -> cycle (2-cycle)
    a, b = ta.copy(), tb.copy()
    y = int(non_min[8])
    a[y], b[y] = tb[x], ta[x]
    assert oracle.check_forest(nindex, nlist, labels, a, b) == 3


def test_forest_checker_accepts_scipy_spanning_trees():
    """scipy's minimum_spanning_tree (Kruskal) of random weighted graphs is a spanning
    forest by a library routine independent of the oracle."""
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import minimum_spanning_tree
    rng = np.random.default_rng(77)
    for trial in range(40):
        n = int(rng.integers(2, 600))
        m = int(rng.integers(0, 2 * n))
        pairs = {(int(min(a, b)), int(max(a, b))) for a, b in
                 zip(rng.integers(0, n, m), rng.integers(0, n, m)) if a != b}
        nindex, nlist = csr_np(n, sorted(pairs))
        labels, ncc = oracle.bfs(nindex, nlist)
        w = rng.random(len(nlist)) + 1.0
        rows = np.repeat(np.arange(n), np.diff(nindex))
        W = {}
        for r, c, x in zip(rows, nlist, w):
            W[(min(r, c), max(r, c))] = x
        keys = sorted(W)
        A = csr_matrix(([W[k] for k in keys], ([k[0] for k in keys], [k[1] for k in keys])),
                       shape=(n, n))
        T = minimum_spanning_tree(A).tocoo()
        edges = list(zip(T.row.tolist(), T.col.tolist()))
        assert len(edges) == n - ncc
        ta, tb = _slots(n, labels, edges, rng)
        assert oracle.check_forest(nindex, nlist, labels, ta, tb) == 0


# ---- CSR preparation (oracle_build_csr) -----------------------------------------

def test_build_csr_hand_examples():
    # loops dropped, duplicates merged (both orientations), back edges added, rows sorted
    nindex, nlist = oracle.build_csr(5, [3, 1, 1, 2, 3, 4], [1, 3, 1, 0, 1, 4])
    assert nindex.tolist() == [0, 1, 2, 3, 4, 4]
    assert nlist.tolist() == [2, 3, 0, 1]
    nindex, nlist = oracle.build_csr(3, [], [])
    assert nindex.tolist() == [0, 0, 0, 0] and nlist.size == 0
    with pytest.raises(ValueError):
        oracle.build_csr(3, [0], [3])


def test_build_csr_matches_scipy():
    """scipy: A = coo(1) + its transpose, diagonal removed, duplicates summed then binarised,
    canonical (sorted) CSR — a library route independent of the oracle's qsort."""
    from scipy.sparse import coo_matrix
    rng = np.random.default_rng(99)
    for trial in range(60):
        n = int(rng.integers(1, 3000))
        E = int(rng.integers(0, 4 * n))
        a = rng.integers(0, n, E).astype(np.int32)
        b = rng.integers(0, n, E).astype(np.int32)
        if trial % 3 == 0 and E >= 4:     # extra loops and duplicates
            q = E // 4
            a[:q] = b[:q]                     # loops
            a[q:2 * q] = b[2 * q:3 * q]       # reversed duplicates of later pairs
            b[q:2 * q] = a[2 * q:3 * q]
        nindex, nlist = oracle.build_csr(n, a, b)
        A = coo_matrix((np.ones(E), (a, b)), shape=(n, n)).tocsr()
        A = (A + A.T).tolil()
        A.setdiag(0)
        A = A.tocsr()
        A.eliminate_zeros()
        A.sort_indices()
        assert np.array_equal(nindex, A.indptr.astype(np.int64))
        assert np.array_equal(nlist, A.indices.astype(np.int32))

"""Graph readers (ecl_cc_read_mtx / ecl_cc_read_edgelist): host-only C code
in libecl_cc.so, so these run without a GPU.  Pinned against entries written by the test
itself and against scipy.io.mmread."""
import os

import numpy as np
import pytest

import oracle
import paper_conf_hpdc_jaiganeshb18_b200 as ecl


def test_mtx_pattern_with_comments(tmp_path):
    p = tmp_path / "g.mtx"
    p.write_bytes(b"%%MatrixMarket matrix coordinate pattern symmetric\r\n"
                  b"% a comment\n%another\n\n"
                  b"5 5 4\n"
                  b"2 1\n5 3\r\n% mid comment\n3 3\n  4   2  \n")
    n, src, dst = ecl.read_mtx(str(p))
    assert n == 5
    assert src.tolist() == [1, 4, 2, 3] and dst.tolist() == [0, 2, 2, 1]


@pytest.mark.parametrize("field,sym", [("real", "general"), ("integer", "symmetric"),
                                       ("pattern", "general"), ("real", "symmetric")])
def test_mtx_matches_scipy(tmp_path, field, sym):
    from scipy.io import mmread, mmwrite
    from scipy.sparse import coo_matrix
    rng = np.random.default_rng(3)
    n = 300
    E = 900
    a = rng.integers(0, n, E)
    b = rng.integers(0, n, E)
    if sym == "symmetric":
        a, b = np.maximum(a, b), np.minimum(a, b)
    vals = rng.integers(1, 9, E).astype(float if field == "real" else int)
    A = coo_matrix((vals, (a, b)), shape=(n, n))
    A.sum_duplicates()
    p = tmp_path / "g.mtx"
    mmwrite(str(p), A, field=field, symmetry=sym)
    nn, src, dst = ecl.read_mtx(str(p))
    assert nn == n
    B = mmread(str(p)).tocoo()
    # scipy expands symmetric files; compare the undirected edge sets
    mine = {(min(x, y), max(x, y)) for x, y in zip(src.tolist(), dst.tolist())}
    ref = {(min(x, y), max(x, y)) for x, y in zip(B.row.tolist(), B.col.tolist())}
    assert mine == ref
    # and the CSR the paper's preparation gives is scipy's symmetrised pattern
    nidx, nl = oracle.build_csr(nn, src, dst)
    S = (coo_matrix((np.ones(B.nnz), (B.row, B.col)), shape=(n, n)).tocsr())
    S = (S + S.T).tolil()
    S.setdiag(0)
    S = S.tocsr()
    S.eliminate_zeros()
    S.sort_indices()
    assert np.array_equal(nidx, S.indptr) and np.array_equal(nl, S.indices)


def test_mtx_errors(tmp_path):
    bad = tmp_path / "bad.mtx"
    bad.write_text("%%MatrixMarket matrix array real general\n2 2\n1\n2\n3\n4\n")
    with pytest.raises(ecl.EclCCError, match="coordinate"):
        ecl.read_mtx(str(bad))
    bad.write_text("%%MatrixMarket matrix coordinate pattern general\n3 3 2\n1 2\n4 1\n")
    with pytest.raises(ecl.EclCCError, match="out of range"):
        ecl.read_mtx(str(bad))
    bad.write_text("%%MatrixMarket matrix coordinate pattern general\n3 3 2\n1 2\n")
    with pytest.raises(ecl.EclCCError, match="bad entry"):
        ecl.read_mtx(str(bad))
    with pytest.raises(ecl.EclCCError, match="cannot read"):
        ecl.read_mtx(str(tmp_path / "missing.mtx"))


def test_edgelist_snap_format(tmp_path):
    p = tmp_path / "g.txt"
    p.write_text("# Directed graph\n# Nodes: 7 Edges: 4\n0\t3\n3 0\n\n6 6\n2    1\n")
    n, src, dst = ecl.read_edgelist(str(p))
    assert n == 7
    assert src.tolist() == [0, 3, 6, 2] and dst.tolist() == [3, 0, 6, 1]
    p.write_text("0 1\n1 x\n")
    with pytest.raises(ecl.EclCCError, match="bad edge"):
        ecl.read_edgelist(str(p))


def test_edgelist_random_roundtrip(tmp_path):
    rng = np.random.default_rng(8)
    a = rng.integers(0, 100000, 20000)
    b = rng.integers(0, 100000, 20000)
    p = tmp_path / "g.txt"
    np.savetxt(str(p), np.stack([a, b], 1), fmt="%d", header="SNAP style", comments="# ")
    n, src, dst = ecl.read_edgelist(str(p))
    assert n == int(max(a.max(), b.max())) + 1
    assert np.array_equal(src, a) and np.array_equal(dst, b)

"""GPU CSR preparation (ecl_cc_build_csr) vs the oracle's plain qsort builder:
the prepared CSR is unique (rows ascending), so the comparison is bit-exact."""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle
import paper_conf_hpdc_jaiganeshb18_b200 as ecl

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def h():
    with ecl.Handle(0) as handle:
        yield handle


def check(h, n, a, b):
    a = np.asarray(a, dtype=np.int32)
    b = np.asarray(b, dtype=np.int32)
    nidx, nl = h.build_csr(n, torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda())
    torch.cuda.synchronize()
    en, el = oracle.build_csr(n, a, b)
    assert np.array_equal(nidx.cpu().numpy(), en)
    assert np.array_equal(nl.cpu().numpy(), el)
    return nidx, nl


@pytest.mark.parametrize("seed", range(6))
def test_random_lists(h, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 200000))
    E = int(rng.integers(0, 5 * n))
    a = rng.integers(0, n, E)
    b = rng.integers(0, n, E)
    if seed % 2:
        a[: E // 5] = b[: E // 5]                     # loops
        a = np.concatenate([a, b[: E // 3]])          # reversed duplicates
        b = np.concatenate([b, a[: E // 3]])
    check(h, n, a, b)


def test_edge_cases(h):
    check(h, 1, [], [])
    check(h, 4, [], [])
    check(h, 4, [2, 2, 2], [2, 2, 2])                 # loops only -> no entries
    check(h, 3, [0, 1, 0, 1], [1, 0, 1, 0])           # one edge, four times
    check(h, 2 ** 20, [0], [2 ** 20 - 1])             # ragged isolated tail


def test_errors(h):
    with pytest.raises(ecl.EclCCError, match="invalid graph"):
        h.build_csr(4, torch.tensor([0, 1], dtype=torch.int32, device="cuda"),
                    torch.tensor([1, 4], dtype=torch.int32, device="cuda"))
    with pytest.raises(ValueError):
        h.build_csr(4, torch.tensor([0], dtype=torch.int32, device="cuda"),
                    torch.tensor([1, 2], dtype=torch.int32, device="cuda"))


@pytest.mark.parametrize("name,sd", [("C4", 6), ("C5", 9), ("C2", 4)])
def test_config_edge_lists_end_to_end(h, name, sd):
    """A generated graph's undirected edges (one direction each, shuffled, with duplicates)
    rebuild exactly the generator's CSR, and ECL-CC on it matches the oracle."""
    g = gg.make_config(name, seed=3, scale_down=sd, device="cpu")
    nidx, nl = g.numpy()
    rows = np.repeat(np.arange(g.n), np.diff(nidx.astype(np.int64)))
    keep = rows > nl
    a, b = rows[keep], nl[keep]
    rng = np.random.default_rng(1)
    perm = rng.permutation(a.size)
    a, b = a[perm], b[perm]
    flip = rng.random(a.size) < 0.5
    a, b = np.where(flip, b, a), np.where(flip, a, b)
    a = np.concatenate([a, b[:1000]])
    b = np.concatenate([b, a[:1000]])
    gi, gl = check(h, g.n, a, b)
    assert np.array_equal(gi.cpu().numpy(), nidx.astype(np.int64))
    labels = h.run(gi, gl)
    torch.cuda.synchronize()
    expect, _ = oracle.bfs(nidx, nl)
    assert np.array_equal(labels.cpu().numpy(), expect)


def test_mtx_file_to_labels(h, tmp_path):
    from scipy.io import mmwrite
    from scipy.sparse import coo_matrix
    rng = np.random.default_rng(4)
    n, E = 50000, 60000
    A = coo_matrix((np.ones(E), (rng.integers(0, n, E), rng.integers(0, n, E))), shape=(n, n))
    p = tmp_path / "g.mtx"
    mmwrite(str(p), A, field="pattern")
    nn, src, dst = ecl.read_mtx(str(p))
    gi, gl = check(h, nn, src, dst)
    labels = h.run(gi, gl)
    torch.cuda.synchronize()
    en, el = oracle.build_csr(nn, src, dst)
    expect, _ = oracle.bfs(en, el)
    assert np.array_equal(labels.cpu().numpy(), expect)

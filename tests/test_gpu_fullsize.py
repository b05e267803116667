"""Full-size parity at BASELINE.json's sizes, in the launch configuration bench.py times
(default handle options).  Every vertex's label is compared with oracle O1 (BFS) and the
invariants I1-I3 are checked; C5 (Graph500 scale 27, ~4.2e9 entries, int64 offsets) takes
about a minute of single-threaded oracle time on the host."""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle
import paper_conf_hpdc_jaiganeshb18_b200 as ecl

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_full_size_exact(name):
    g = gg.make_config(name, seed=1, device="cuda")
    with ecl.Handle(0) as h:
        out = h.run(g.nindex, g.nlist)
        out2 = h.run(g.nindex, g.nlist)          # second run on the reused scratch
        torch.cuda.synchronize()
    got = out.cpu().numpy()
    assert np.array_equal(got, out2.cpu().numpy())
    nidx, nl = g.numpy()
    del g, out, out2
    torch.cuda.empty_cache()
    expect, ncc = oracle.bfs(nidx, nl)
    bad = np.nonzero(got != expect)[0]
    assert bad.size == 0, f"{name}: {bad.size} labels differ (first v={bad[0]})"
    assert oracle.check(nidx, nl, got, ncc) == 0


_EXPECT = {}


def _expect(name, g):
    if name not in _EXPECT:
        nidx, nl = g.numpy()
        _EXPECT[name] = oracle.bfs(nidx, nl)
    return _EXPECT[name]


@pytest.mark.parametrize("name", ["C3", "C4", "C5"])
def test_full_size_option_variants(name):
    """The same full-size graphs under the non-default memory model and kernel paths:
    load_mode 0 (every racing parent[] load ld.relaxed.gpu, SURVEY R7 as written;
    DESIGN.md §5 "Memory model"), the paper's sequential kernel order 0, and the
    R31 16-byte quad engine."""
    g = gg.make_config(name, seed=1, device="cuda")
    expect, ncc = _expect(name, g)
    variants = [{"load_mode": 0}, {"order": 0}, {"vec": 1}, {"vec": 0},
                {"load_mode": 0, "order": 0}]
    with ecl.Handle(0) as h:
        for opts in variants:
            for k, v in opts.items():
                h.set_option(k, v)
            got = h.run(g.nindex, g.nlist).cpu().numpy()
            for k in opts:
                h.set_option(k, {"load_mode": 1, "order": 2, "vec": 2}[k])
            bad = np.nonzero(got != expect)[0]
            assert bad.size == 0, f"{name} {opts}: {bad.size} labels differ (first v={bad[0]})"
    nidx, nl = g.numpy()
    assert oracle.check(nidx, nl, got, ncc) == 0

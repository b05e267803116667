"""GPU parity of the R33 single-launch path (R33, ECL_CC_OPT_FUSED): the whole
ECL-CC path (locality probe, init_bin, depth probe + R23 passes, the three hook kernels,
finalize) as ONE cooperative grid with grid barriers between the phases.  Labels must
equal oracle O1 on every graph family and option the multi-kernel path supports,
and the auto mode must pick the single launch exactly for small graphs."""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle
import paper_conf_hpdc_jaiganeshb18_b200 as ecl

pytestmark = pytest.mark.gpu

SMALL = {"C1": 0, "C2": 4, "C3": 4, "C4": 6, "C5": 10}
RESET = {"fused": 2, "order": 2, "filter": 2, "prejump": 2, "jump": 4, "init": 3, "fini": 3,
         "batch": 1, "load_mode": 1, "grid_blocks": 0, "fuse_init": 2, "stop_after": 0,
         "thresh_thread": 16, "thresh_warp": 352}


@pytest.fixture(scope="module")
def h():
    with ecl.Handle(0) as handle:
        yield handle


def run(h, g, index_dtype=None, **opts):
    g = g.to("cuda")
    nindex = g.nindex if index_dtype is None else g.nindex.to(index_dtype)
    for k, v in opts.items():
        h.set_option(k, v)
    try:
        out = h.run(nindex, g.nlist)
        torch.cuda.synchronize()
        fused = h.run_info()["fused"]
    finally:
        for k in opts:
            h.set_option(k, RESET[k])
    return out.cpu().numpy(), fused


def check(h, g, **opts):
    nidx, nl = g.numpy()
    expect, ncc = oracle.bfs(nidx, nl)
    got, fused = run(h, g, **opts)
    assert np.array_equal(got, expect), f"{g.name} {opts}"
    assert oracle.check(nidx, nl, got, ncc) == 0
    return fused


def hand():
    from test_gpu_parity import hand_graphs
    from test_gpu_raw_csr import hand_raw_graphs
    return hand_graphs() + hand_raw_graphs()


@pytest.mark.parametrize("g", hand(), ids=lambda g: g.name)
def test_fused_hand_built(h, g):
    assert check(h, g, fused=1)


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("seed", [1, 2])
def test_fused_configs(h, name, seed):
    g = gg.make_config(name, seed=seed, scale_down=SMALL[name])
    assert check(h, g, fused=1)


@pytest.mark.parametrize("opts", [dict(prejump=1), dict(prejump=0), dict(filter=1),
                                  dict(fuse_init=1), dict(fuse_init=0), dict(load_mode=0),
                                  dict(jump=1), dict(jump=2), dict(jump=3), dict(batch=0),
                                  dict(init=1, fini=1), dict(init=2, fini=2),
                                  dict(thresh_thread=2, thresh_warp=20), dict(grid_blocks=3),
                                  dict(grid_blocks=148)],
                         ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
@pytest.mark.parametrize("name", ["C1", "C2", "C4"])
def test_fused_options(h, name, opts):
    g = gg.make_config(name, seed=3, scale_down=max(SMALL[name], 2))
    assert check(h, g, fused=1, **opts)


def test_fused_int64_and_raw(h):
    g = gg.inject_loops_dups(gg.make_config("C4", seed=4, scale_down=7), seed=3)
    nidx, nl = g.numpy()
    expect, _ = oracle.bfs(nidx, nl)
    got, fused = run(h, g, index_dtype=torch.int64, fused=1)
    assert fused and np.array_equal(got, expect)


def test_fused_unflattened_forest(h):
    # STOP_AFTER 2: the forest is left unflattened; every parent is a same-component
    # vertex no larger than the child, and flattening it gives the labels
    g = gg.make_config("C1", seed=5)
    nidx, nl = g.numpy()
    expect, _ = oracle.bfs(nidx, nl)
    par, fused = run(h, g, fused=1, stop_after=2)
    assert fused
    v = np.arange(g.n)
    assert np.all(par <= v) and np.array_equal(expect[par], expect)


def test_fused_spanning_forest(h):
    g = gg.make_config("C1", seed=6)
    gd = g.to("cuda")
    h.set_option("fused", 1)
    try:
        lab, ta, tb = h.spanning_forest(gd.nindex, gd.nlist)
        torch.cuda.synchronize()
    finally:
        h.set_option("fused", 2)
    nidx, nl = g.numpy()
    expect, _ = oracle.bfs(nidx, nl)
    assert np.array_equal(lab.cpu().numpy(), expect)
    assert oracle.check_forest(nidx, nl, expect, ta.cpu().numpy(), tb.cpu().numpy()) == 0


def test_fused_auto_choice(h):
    small = gg.make_config("C1", seed=1)
    assert check(h, small) is True                      # auto: C1 takes the single launch
    big = gg.make_config("C4", seed=1, scale_down=4)    # 2^20 rows, 2^25 entries: above
    assert check(h, big) is False
    assert check(h, small, fused=0) is False


def test_fused_repeat_and_stream(h):
    g = gg.make_config("C1", seed=7).to("cuda")
    s = torch.cuda.Stream()
    h.set_option("fused", 1)
    try:
        with torch.cuda.stream(s):
            outs = [h.run(g.nindex, g.nlist, stream=s) for _ in range(3)]
        s.synchronize()
    finally:
        h.set_option("fused", 2)
    expect, _ = oracle.bfs(*g.numpy())
    for o in outs:
        assert np.array_equal(o.cpu().numpy(), expect)


def test_fused_and_vec_option_values(h):
    # ECL_CC_OPT_FUSED / ECL_CC_OPT_VEC take 0, 1 or 2; anything else is INVALID_ARG
    for name in ("fused", "vec"):
        for bad in (-1, 3):
            with pytest.raises(ecl.EclCCError):
                h.set_option(name, bad)
        for ok in (0, 1, 2):
            h.set_option(name, ok)
        h.set_option(name, 2)

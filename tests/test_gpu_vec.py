"""GPU parity of the R31 quad engine (R31): hook_warp / hook_block stream the
adjacency as aligned 16-byte quads, masking the entries of a piece's first and last quad
that belong to neighbouring rows.  The labels must equal oracle O1 whatever the
alignment of the rows, with the engine on or off (ECL_CC_OPT_VEC), with a misaligned
adjacency base (the host then falls back to four-byte loads), and when the last quad of
nlist is partial (m % 4 != 0: no over-read past the caller's buffer).
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


def run_opts(h, nindex, nlist, **opts):
    for k, v in opts.items():
        h.set_option(k, v)
    try:
        out = h.run(nindex, nlist)
        torch.cuda.synchronize()
    finally:
        h.set_option("vec", 2).set_option("order", 2).set_option("filter", 2)
        h.set_option("thresh_thread", 16).set_option("thresh_warp", 352)
    return out.cpu().numpy()


def expect_of(g):
    nidx, nl = g.numpy()
    return oracle.bfs(nidx, nl)


def misaligned(nlist, shift):
    """The same entries at a base `shift` ints past a 16-byte boundary."""
    buf = torch.empty(nlist.numel() + 4, dtype=nlist.dtype, device=nlist.device)
    view = buf[shift:shift + nlist.numel()]
    view.copy_(nlist)
    assert view.data_ptr() % 16 == 4 * shift
    return view


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("vec", [0, 1, 2])
@pytest.mark.parametrize("order", [0, 2])
def test_vec_configs(h, name, vec, order):
    g = gg.make_config(name, seed=3, scale_down=SMALL[name], device="cuda")
    expect, ncc = expect_of(g)
    got = run_opts(h, g.nindex, g.nlist, vec=vec, order=order)
    assert np.array_equal(got, expect), f"{name} vec={vec} order={order}"
    nidx, nl = g.numpy()
    assert oracle.check(nidx, nl, got, ncc) == 0


@pytest.mark.parametrize("name", ["C3", "C4", "C5"])
@pytest.mark.parametrize("shift", [1, 2, 3])
def test_vec_misaligned_base(h, name, shift):
    g = gg.make_config(name, seed=5, scale_down=SMALL[name], device="cuda")
    expect, _ = expect_of(g)
    got = run_opts(h, g.nindex, misaligned(g.nlist, shift), vec=1)
    assert np.array_equal(got, expect)


@pytest.mark.parametrize("t1,t2", [(0, 0), (0, 10**9), (2, 5), (3, 40)])
@pytest.mark.parametrize("filt", [0, 1])
def test_vec_every_row_in_range_kernels(h, t1, t2, filt):
    # low thresholds push short rows (1..5 entries) into hook_warp / hook_block, so pieces
    # start and end inside one quad and several pieces share a quad
    g = gg.make_config("C4", seed=7, scale_down=7, device="cuda")
    expect, _ = expect_of(g)
    got = run_opts(h, g.nindex, g.nlist, vec=1, thresh_thread=t1, thresh_warp=t2, filter=filt)
    assert np.array_equal(got, expect)


@pytest.mark.parametrize("tail", [1, 2, 3])
def test_vec_partial_last_quad(h, tail):
    # a hub as the LAST row, with m % 4 == tail: its last quad ends at the buffer's end
    n = 3000
    hub = n - 1
    pairs = [(hub, i) for i in range(0, n - 1, 2)] + [(i, i + 1) for i in range(1, n - 2, 4)]
    loops = [hub] * ((tail - 2 * len(pairs)) % 4)     # the hub's loops end its row
    R = [a for a, b in pairs] + [b for a, b in pairs] + loops
    C = [b for a, b in pairs] + [a for a, b in pairs] + loops
    g = gg.raw_csr(f"hub_last_{tail}", n, torch.tensor(R), torch.tensor(C))
    nindex, nlist = g.nindex.to("cuda"), g.nlist.to("cuda")
    m = nlist.numel()
    assert m % 4 == tail
    exact = torch.empty(m, dtype=nlist.dtype, device="cuda")   # no slack after the end
    exact.copy_(nlist)
    expect, _ = expect_of(g)
    got = run_opts(h, nindex, exact, vec=1, thresh_thread=1, thresh_warp=4)
    assert np.array_equal(got, expect), f"m={m}"


def test_vec_raw_csr_loops_dups(h):
    g = gg.inject_loops_dups(gg.make_config("C4", seed=2, scale_down=6, device="cuda"), seed=9)
    expect, _ = expect_of(g)
    for vec in (0, 1):
        got = run_opts(h, g.nindex, g.nlist, vec=vec, thresh_thread=2, thresh_warp=20)
        assert np.array_equal(got, expect)


def test_vec_int64_offsets(h):
    g = gg.make_config("C5", seed=4, scale_down=9, device="cuda")
    expect, _ = expect_of(g)
    got = run_opts(h, g.nindex.to(torch.int64), misaligned(g.nlist, 0), vec=1)
    assert np.array_equal(got, expect)

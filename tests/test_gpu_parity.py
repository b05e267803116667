"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

The min-ID labelling is unique (R13), so every comparison is element-by-element
equality with oracle O1 (BFS), plus the invariants I1-I3 on the GPU output.
"""
import itertools

import numpy as np
import pytest
import torch

import graphgen as gg
import oracle
import paper_conf_hpdc_jaiganeshb18_b200 as ecl

pytestmark = pytest.mark.gpu

DEFAULTS = {"thresh_thread": 16, "thresh_warp": 352, "load_mode": 1, "ttas": 1, "init": 3,
            "jump": 4, "fini": 3, "batch": 1, "filter": 2, "order": 2, "prejump": 2,
            "fuse_init": 2, "flatten_passes": 0}


@pytest.fixture(scope="module")
def h():
    with ecl.Handle(0) as handle:
        yield handle


def gpu_labels(h, g, index_dtype=None, **opts):
    g = g.to("cuda")
    nindex = g.nindex if index_dtype is None else g.nindex.to(index_dtype)
    for k, v in opts.items():
        h.set_option(k, v)
    try:
        out = h.run(nindex, g.nlist)
        torch.cuda.synchronize()
    finally:
        for k in opts:
            h.set_option(k, DEFAULTS.get(k, 0))
    return out.cpu().numpy()


def assert_parity(h, g, **kw):
    nidx, nl = g.numpy()
    expect, ncc = oracle.bfs(nidx, nl)
    got = gpu_labels(h, g, **kw)
    if not np.array_equal(got, expect):
        bad = np.nonzero(got != expect)[0]
        raise AssertionError(f"{g.name}: {len(bad)} of {g.n} labels differ, first at v={bad[0]}: "
                             f"gpu {got[bad[0]]} oracle {expect[bad[0]]}")
    assert oracle.check(nidx, nl, got, ncc) == 0
    return ncc


# ---------------------------------------------------------------------------------------
# hand-built graphs
# ---------------------------------------------------------------------------------------
def hand_graphs():
    G = []
    G.append(gg.from_edges(1, [], "single"))
    G.append(gg.from_edges(7, [], "no_edges"))
    G.append(gg.from_edges(5, [(4, 2), (2, 0), (0, 3), (3, 1)], "scrambled_path"))
    ev = [(a, b) for a in range(0, 40, 2) for b in range(a + 2, 40, 2)]
    od = [(a, b) for a in range(1, 40, 2) for b in range(a + 2, 40, 2)]
    G.append(gg.from_edges(40, ev + od, "interleaved_cliques"))
    G.append(gg.from_edges(10, [(3, 6), (7, 8), (6, 8)], "fig2"))
    n = 5000
    G.append(gg.from_edges(n, [(n - 1, i) for i in range(n - 1)], "star_center_last"))
    G.append(gg.from_edges(n, [(0, i) for i in range(1, n)], "star_center_0"))
    G.append(gg.from_edges(400, list(itertools.combinations(range(400), 2)), "K400"))
    # rows of degree exactly 16 / 17 / 352 / 353 around the bin thresholds
    edges = []
    base = 0
    for d in (15, 16, 17, 18, 351, 352, 353, 354):
        hub = base + d  # hub has the largest ID so it is active and hooks all its leaves
        edges += [(hub, base + i) for i in range(d)]
        base += d + 1
    G.append(gg.from_edges(base, edges, "degree_boundaries"))
    # same, hubs with the smallest ID (inactive hubs: leaves hook into them)
    edges = []
    base = 0
    for d in (16, 17, 352, 353):
        edges += [(base, base + 1 + i) for i in range(d)]
        base += d + 1
    G.append(gg.from_edges(base, edges, "degree_boundaries_lowhub"))
    return G


@pytest.mark.parametrize("g", hand_graphs(), ids=lambda g: g.name)
def test_hand_built(h, g):
    assert_parity(h, g)


def test_empty_graph(h):
    out = h.run(torch.zeros(1, dtype=torch.int32, device="cuda"),
                torch.zeros(0, dtype=torch.int32, device="cuda"))
    assert out.numel() == 0


def test_big_hub_chunked(h):
    """One hub with 1.5M neighbours (spread over many warps), plus a second component."""
    n = 1_500_002
    src = torch.full((n - 2,), n - 2, dtype=torch.int64)
    dst = torch.arange(n - 2, dtype=torch.int64)
    g = gg.csr_from_pairs("hub1.5M", n, src, dst)
    assert assert_parity(h, g) == 2


def test_reversed_long_chain(h):
    n = 1 << 20
    v = torch.arange(1, n, dtype=torch.int64)
    g = gg.csr_from_pairs("chain", n, v, v - 1)
    assert assert_parity(h, g) == 1


def test_fig3_pointer_jumping_shape(h):
    """Long paths under Init3: a path whose IDs increase along it (each v's first smaller
    neighbour is v-1), plus a path with IDs decreasing from the middle outwards."""
    n = 100_000
    a = list(range(0, n // 2 - 1))
    e = [(i + 1, i) for i in a] + [(n // 2 + i, n // 2 + i + 1) for i in range(n // 2 - 1)]
    e.append((n // 2, 0))
    assert assert_parity(h, gg.from_edges(n, e, "two_paths")) == 1


# ---------------------------------------------------------------------------------------
# the five BASELINE configs, scaled so the oracle finishes in seconds
# ---------------------------------------------------------------------------------------
SMALL = {"C1": 0, "C2": 4, "C3": 4, "C4": 6, "C5": 10}


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("seed", [1, 2])
def test_configs_scaled(h, name, seed):
    g = gg.make_config(name, seed=seed, scale_down=SMALL[name], device="cuda")
    assert_parity(h, g)


@pytest.mark.parametrize("name", ["C1", "C3", "C4"])
def test_row_shuffle_order_independence(h, name):
    g = gg.make_config(name, seed=3, scale_down=SMALL[name], device="cuda")
    assert_parity(h, gg.shuffle_rows(g, seed=5))


@pytest.mark.parametrize("grid", [1, 3, 148, 2000])
@pytest.mark.parametrize("mode", [0, 1])
def test_launch_config_sweep(h, grid, mode):
    """Race shaking: very different interleavings must give the same labels."""
    g = gg.make_config("C4", seed=4, scale_down=8, device="cuda")
    assert_parity(h, g, grid_blocks=grid, load_mode=mode)


@pytest.mark.parametrize("t1,t2", [(0, 0), (0, 10**9), (4, 8), (16, 352), (10**9, 10**9)])
def test_threshold_sweep(h, t1, t2):
    g = gg.make_config("C4", seed=5, scale_down=8, device="cuda")
    assert_parity(h, g, thresh_thread=t1, thresh_warp=t2)


@pytest.mark.parametrize("name", ["C2", "C4"])
def test_int64_offsets(h, name):
    g = gg.make_config(name, seed=1, scale_down=SMALL[name], device="cuda")
    assert_parity(h, g, index_dtype=torch.int64)


# ---------------------------------------------------------------------------------------
# intermediate, deterministic stages
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("name", ["C1", "C4"])
def test_init3_stage(h, name):
    """stop_after=1 leaves Init3's parents in the output: exact per vertex."""
    g = gg.make_config(name, seed=2, scale_down=SMALL[name], device="cuda")
    g = gg.shuffle_rows(g, seed=9)
    got = gpu_labels(h, g, stop_after=1)
    assert np.array_equal(got, oracle.init3(*g.numpy()))


def test_worklist_sets(h):
    """Bins (reading R2/R3): front = active with 16 < deg <= 352, back = deg > 352
    (the separate Init3 pass; with R28 the bins hold every row of the degree range)."""
    g = gg.make_config("C4", seed=1, scale_down=4, device="cuda")
    gpu_labels(h, g, fuse_init=0)
    front, back = h.worklist()
    nidx, nl = g.numpy()
    deg = np.diff(nidx.astype(np.int64))
    active = oracle.init3(nidx, nl) != np.arange(g.n)
    ef = np.nonzero(active & (deg > 16) & (deg <= 352))[0]
    eb = np.nonzero(active & (deg > 352))[0]
    assert np.array_equal(np.sort(front.cpu().numpy()), ef)
    assert np.array_equal(np.sort(back.cpu().numpy()), eb)
    gpu_labels(h, g, fuse_init=1)                     # R28: degree-only bins
    front, back = h.worklist()
    assert np.array_equal(np.sort(front.cpu().numpy()), np.nonzero((deg > 16) & (deg <= 352))[0])
    assert np.array_equal(np.sort(back.cpu().numpy()), np.nonzero(deg > 352)[0])


def test_run_host_end_to_end(h):
    g = gg.make_config("C3", seed=1, scale_down=6)
    nidx, nl = g.numpy()
    out = h.run_host(torch.from_numpy(nidx).pin_memory(), torch.from_numpy(nl).pin_memory())
    expect, _ = oracle.bfs(nidx, nl)
    assert np.array_equal(out.numpy(), expect)


def test_non_default_stream(h):
    g = gg.make_config("C3", seed=2, scale_down=6, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        out = h.run(g.nindex, g.nlist)
    s.synchronize()
    expect, _ = oracle.bfs(*g.numpy())
    assert np.array_equal(out.cpu().numpy(), expect)


def test_argument_errors(h):
    idx = torch.zeros(5, dtype=torch.int32, device="cuda")
    with pytest.raises(TypeError):
        h.run(idx.float(), torch.zeros(0, dtype=torch.int32, device="cuda"))
    lib = h._lib
    assert lib.ecl_cc_run(h._h, -1, 0, None, None, None, None) == 1
    assert lib.ecl_cc_run(h._h, 4, 2**31, idx.data_ptr(), None, None, None) == 1
    assert lib.ecl_cc_run(h._h, 0, 0, None, None, None, None) == 0
    for bad in (-1, 3):                       # kernel orders are 0, 1, 2
        with pytest.raises(ecl.EclCCError, match="order"):
            h.set_option("order", bad)


def test_validate(h):
    g = gg.make_config("C1", seed=1, scale_down=4, device="cuda")
    assert h.validate(g.nindex, g.nlist)
    asym = gg.Graph("asym", 3, torch.tensor([0, 1, 1, 1], dtype=torch.int32, device="cuda"),
                    torch.tensor([2], dtype=torch.int32, device="cuda"))
    assert not h.validate(asym.nindex, asym.nlist)
    bad = gg.Graph("oob", 2, torch.tensor([0, 1, 1], dtype=torch.int32, device="cuda"),
                   torch.tensor([7], dtype=torch.int32, device="cuda"))
    assert not h.validate(bad.nindex, bad.nlist)


def test_stats_identity():
    """-DECL_CC_STATS build: each successful hook CAS removes exactly one root, and
    halving stores never create one, so #successful CAS == #Init3 roots - #CC (§8c).
    With R28 (Init3 folded into the hook kernels) the forest starts as n roots and the
    Init CASes count too: #successful CAS == n - #CC."""
    with ecl.Handle(0, stats=True) as hs:
        assert hs.stats_enabled
        for name in ("C1", "C3", "C4"):
            g = gg.make_config(name, seed=1, scale_down=SMALL[name], device="cuda")
            nidx, nl = g.numpy()
            expect, ncc = oracle.bfs(nidx, nl)
            roots = int((oracle.init3(nidx, nl) == np.arange(g.n)).sum())
            for fuse, start in ((0, roots), (1, g.n)):
                got = gpu_labels(hs, g, fuse_init=fuse)
                st = hs.stats()
                assert np.array_equal(got, expect)
                assert st["cas_success"] == start - ncc, (name, fuse, st, start, ncc)


def test_pre_finalize_forest_invariant(h):
    """Before Fini3 every parent[x] <= x and the forest's roots are the component minima."""
    g = gg.make_config("C3", seed=1, scale_down=6, device="cuda")
    par = gpu_labels(h, g, stop_after=2)
    assert np.all(par <= np.arange(g.n))
    expect, ncc = oracle.bfs(*g.numpy())
    assert int((par == np.arange(g.n)).sum()) == ncc


# ---------------------------------------------------------------------------------------
# multi-GPU math on one device: row partitions -> local forests -> sequential merges
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("G", [1, 2, 3, 4, 8])
def test_fake_multi_gpu_merge(h, G):
    from paper_conf_hpdc_jaiganeshb18_b200 import dist
    g = gg.make_config("C4", seed=2, scale_down=7, device="cuda")
    expect, _ = oracle.bfs(*g.numpy())
    nindex64 = g.nindex.to(torch.int64)
    bounds = dist.partition_rows(nindex64.cpu(), G)
    forests = []
    for r in range(G):
        lo, hi = bounds[r], bounds[r + 1]
        idx, lst = dist.slice_rows(nindex64, g.nlist, lo, hi)
        forests.append(h.run_rows(g.n, lo, hi, idx, lst))
    acc = forests[0]
    for f in forests[1:]:
        h.merge(acc, f)
    h.finalize(acc)
    torch.cuda.synchronize()
    assert np.array_equal(acc.cpu().numpy(), expect)


@pytest.mark.parametrize("G", [2, 3, 8])
@pytest.mark.parametrize("name", ["C2", "C4", "C5"])
def test_fake_multi_gpu_unflattened_tree_merge(h, name, G):
    """dist.forest_merge's schedule on one GPU: work-weighted partition, unflattened local
    forests (flatten=False), binomial-tree merges, one flatten at the end."""
    from paper_conf_hpdc_jaiganeshb18_b200 import dist
    g = gg.make_config(name, seed=4, scale_down=SMALL[name] + 1, device="cuda")
    expect, _ = oracle.bfs(*g.numpy())
    nindex64 = g.nindex.to(torch.int64)
    bounds = dist.partition_rows(nindex64, G, weights=dist.row_weights(nindex64, g.nlist))
    forests = []
    for r in range(G):
        idx, lst = dist.slice_rows(nindex64, g.nlist, bounds[r], bounds[r + 1])
        forests.append(h.run_rows(g.n, bounds[r], bounds[r + 1], idx, lst, flatten=False))
    for (_, send, recv) in dist.tree_schedule(G):
        chunks = [(c * g.n) // 3 for c in range(4)]
        for c in range(3):
            h.merge(forests[recv], forests[send][chunks[c]:chunks[c + 1]], chunks[c])
    h.finalize(forests[0])
    torch.cuda.synchronize()
    assert np.array_equal(forests[0].cpu().numpy(), expect)


# ---------------------------------------------------------------------------------------
# paper ablations: every Init/Jump/Fini variant must give the same labels
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("init", [1, 2, 3])
@pytest.mark.parametrize("jump", [1, 2, 3, 4])
@pytest.mark.parametrize("fini", [1, 2, 3])
@pytest.mark.parametrize("name", ["C2", "C4"])
def test_ablation_variants(h, name, init, jump, fini):
    g = gg.make_config(name, seed=6, scale_down={"C2": 6, "C4": 8}[name], device="cuda")
    g = gg.shuffle_rows(g, seed=2)
    assert_parity(h, g, init=init, jump=jump, fini=fini)


@pytest.mark.parametrize("init", [1, 2])
def test_init_variant_stage(h, init):
    """Init1 leaves parent[v] = v; Init2 the smallest neighbour if smaller."""
    g = gg.shuffle_rows(gg.make_config("C4", seed=3, scale_down=8, device="cuda"), seed=4)
    got = gpu_labels(h, g, stop_after=1, init=init)
    nidx, nl = g.numpy()
    if init == 1:
        assert np.array_equal(got, np.arange(g.n))
    else:
        deg = np.diff(nidx.astype(np.int64))
        rows = np.repeat(np.arange(g.n), deg)
        mn = np.arange(g.n)
        np.minimum.at(mn, rows, nl)
        assert np.array_equal(got, mn)


# ---------------------------------------------------------------------------------------
# R21 anchor-tree membership filter (forced on at small sizes; auto-on only for 4n > 128 MB)
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("grid", [0, 3, 148])
def test_membership_filter(h, name, grid):
    g = gg.make_config(name, seed=8, scale_down=SMALL[name], device="cuda")
    assert_parity(h, g, filter=1, grid_blocks=grid)


@pytest.mark.parametrize("mode", [0, 1, 2, 3])
def test_load_modes_with_filter(h, mode):
    g = gg.make_config("C5", seed=9, scale_down=9, device="cuda")
    assert_parity(h, g, filter=1, load_mode=mode)


# ---------------------------------------------------------------------------------------
# kernel order option (hubs first): same labels
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("name", list(SMALL))
def test_order_hubs_first(h, name):
    g = gg.make_config(name, seed=12, scale_down=SMALL[name], device="cuda")
    assert_parity(h, g, order=1)
    assert_parity(h, g, order=1, filter=1)
    assert_parity(h, g, order=0)                  # the paper's order
    assert_parity(h, g, order=0, filter=1)


@pytest.mark.parametrize("name", list(SMALL))
def test_order_concurrent(h, name):
    # hook_block on a side stream next to hook_warp + hook_thread (order 2): the three
    # kernels hook the same edge sets concurrently; Fig. 6 is order-free (R13)
    g = gg.make_config(name, seed=13, scale_down=SMALL[name], device="cuda")
    assert_parity(h, g, order=2)
    assert_parity(h, g, order=2, filter=1)
    assert_parity(h, g, order=2, filter=1, occ_range=2, occ_thread=6)
    assert_parity(h, g, order=2, filter=1, occ_range=8)


# ---------------------------------------------------------------------------------------
# spanning forest: labels bit-exact, forest valid by the oracle's checker
# (the forest itself is one of many valid answers)
# ---------------------------------------------------------------------------------------
def assert_forest(h, g, index_dtype=None, **opts):
    g = g.to("cuda")
    nindex = g.nindex if index_dtype is None else g.nindex.to(index_dtype)
    for k, v in opts.items():
        h.set_option(k, v)
    try:
        lab, ta, tb = h.spanning_forest(nindex, g.nlist)
        torch.cuda.synchronize()
    finally:
        for k in opts:
            h.set_option(k, DEFAULTS.get(k, 0))
    nidx, nl = g.numpy()
    expect, ncc = oracle.bfs(nidx, nl)
    lab = lab.cpu().numpy()
    assert np.array_equal(lab, expect), f"{g.name}: labels differ"
    rc = oracle.check_forest(nidx, nl, expect, ta.cpu().numpy(), tb.cpu().numpy())
    assert rc == 0, f"{g.name}: forest check failed with code {rc}"


@pytest.mark.parametrize("g", hand_graphs(), ids=lambda g: g.name)
def test_forest_hand_built(h, g):
    assert_forest(h, g)


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("seed", [1, 2])
def test_forest_configs(h, name, seed):
    g = gg.make_config(name, seed=seed, scale_down=SMALL[name], device="cuda")
    assert_forest(h, g)
    assert_forest(h, gg.shuffle_rows(g, seed=seed + 10))


@pytest.mark.parametrize("opts", [dict(filter=1), dict(order=1), dict(ttas=0),
                                  dict(init=1), dict(init=2), dict(jump=1), dict(jump=3),
                                  dict(batch=0), dict(grid_blocks=3), dict(load_mode=0)],
                         ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
def test_forest_variants(h, opts):
    g = gg.make_config("C4", seed=5, scale_down=8, device="cuda")
    assert_forest(h, g, **opts)
    assert_forest(h, gg.make_config("C2", seed=5, scale_down=6, device="cuda"), **opts)


def test_forest_int64_offsets(h):
    g = gg.make_config("C5", seed=4, scale_down=9, device="cuda")
    assert_forest(h, g, index_dtype=torch.int64)


# ---------------------------------------------------------------------------------------
# R23 pointer-doubling passes between init and the hook kernels: forced on, forced off,
# auto (default) — same labels; the grid configs (deep Init3 forests) trigger auto mode
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("prejump", [0, 1])
def test_prejump_configs(h, name, prejump):
    g = gg.make_config(name, seed=21, scale_down=SMALL[name], device="cuda")
    assert_parity(h, g, prejump=prejump)


@pytest.mark.parametrize("g", hand_graphs(), ids=lambda g: g.name)
def test_prejump_hand_built(h, g):
    assert_parity(h, g, prejump=1)


@pytest.mark.parametrize("prejump", [1, 2])
def test_prejump_long_chains(h, prejump):
    n = 1 << 20
    v = torch.arange(1, n, dtype=torch.int64)
    assert assert_parity(h, gg.csr_from_pairs("chain", n, v, v - 1), prejump=prejump) == 1
    g = gg.make_config("C2", seed=3, scale_down=2, device="cuda")
    assert_parity(h, g, prejump=prejump, filter=1)
    assert_parity(h, g, prejump=prejump, jump=2, init=2)


# ---------------------------------------------------------------------------------------
# CUDA graph capture: ecl_cc_run only enqueues work on the caller's stream (the order-2
# side stream is forked from and joined back into it with events), so a whole run can be
# captured once and replayed; replays must give the oracle's labels every time
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("name,order", [("C4", 2), ("C4", 0), ("C2", 2), ("C5", 2)])
def test_cuda_graph_capture_replay(h, name, order):
    g = gg.make_config(name, seed=21, scale_down=SMALL[name], device="cuda")
    nidx, nl = g.numpy()
    expect, _ = oracle.bfs(nidx, nl)
    h.set_option("order", order)     # C2 also captures R23's cooperative pass kernel
    try:
        out = torch.empty(g.n, dtype=torch.int32, device="cuda")
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            h.run(g.nindex, g.nlist, out=out)     # warm-up: grows the handle's scratch
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=s):
            h.run(g.nindex, g.nlist, out=out)
        for _ in range(3):
            out.fill_(-1)
            graph.replay()
            torch.cuda.synchronize()
            assert np.array_equal(out.cpu().numpy(), expect)
    finally:
        h.set_option("order", DEFAULTS["order"])


# ---------------------------------------------------------------------------------------
# encoded forest exchange: encode each fake rank's flattened forest,
# merge all encodings into rank 0's forest in one call, flatten once
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("G", [2, 3, 5, 9])
@pytest.mark.parametrize("name", ["C2", "C4", "C5"])
def test_fake_multi_gpu_encoded_merge(h, name, G):
    from paper_conf_hpdc_jaiganeshb18_b200 import dist
    g = gg.make_config(name, seed=7, scale_down=SMALL[name] + 1, device="cuda")
    expect, _ = oracle.bfs(*g.numpy())
    nindex64 = g.nindex.to(torch.int64)
    bounds = dist.partition_rows(nindex64, G, weights=dist.row_weights(nindex64, g.nlist))
    forests, encs = [], []
    for r in range(G):
        idx, lst = dist.slice_rows(nindex64, g.nlist, bounds[r], bounds[r + 1])
        f = h.run_rows(g.n, bounds[r], bounds[r + 1], idx, lst, flatten=(r > 0))
        forests.append(f)
        if r > 0:
            enc = h.encode_buffers(g.n)
            h.forest_encode(f, dist.row_anchor(idx, bounds[r]), enc)
            encs.append(enc)
    h.merge_encoded(forests[0], encs)
    h.finalize(forests[0])
    torch.cuda.synchronize()
    assert np.array_equal(forests[0].cpu().numpy(), expect)


def test_forest_encode_exact(h):
    """The encoding of a flattened labelling: bitmap = {v : L[v] == L[anchor]}, pairs =
    {(v, L[v]) : L[v] != v, L[v] != D}, meta = (#pairs, D)."""
    g = gg.make_config("C4", seed=8, scale_down=8, device="cuda")
    lab = h.run(g.nindex, g.nlist)
    anchor = int(torch.argmax(g.degrees()))
    enc = h.encode_buffers(g.n)
    h.forest_encode(lab, anchor, enc)
    torch.cuda.synchronize()
    L = lab.cpu().numpy()
    D = L[anchor]
    meta = enc["meta"].cpu().numpy()
    assert meta[1] == D
    v = np.arange(g.n)
    want_pairs = set(zip(v[(L != v) & (L != D)].tolist(), L[(L != v) & (L != D)].tolist()))
    P = enc["pairs"].cpu().numpy()[:2 * meta[0]].reshape(-1, 2)
    assert meta[0] == len(want_pairs) and set(map(tuple, P.tolist())) == want_pairs
    bits = enc["bits"].cpu().numpy().view(np.uint32)
    got = (bits[v // 32] >> (v % 32)) & 1
    assert np.array_equal(got.astype(bool), L == D)
    # merging the encoding into an identity forest and flattening reproduces the labels
    par = torch.arange(g.n, dtype=torch.int32, device="cuda")
    h.merge_encoded(par, [enc])
    h.finalize(par)
    assert np.array_equal(par.cpu().numpy(), L)


def test_forest_encode_small_cap(h):
    """meta[0] reports the needed pair count when cap is too small (only cap written)."""
    g = gg.make_config("C1", seed=9, device="cuda")
    lab = h.run(g.nindex, g.nlist)
    enc = h.encode_buffers(g.n, cap=3)
    h.forest_encode(lab, 0, enc)
    L = lab.cpu().numpy()
    D = L[0]
    v = np.arange(g.n)
    assert int(enc["meta"][0]) == int(((L != v) & (L != D)).sum()) > 3


@pytest.mark.parametrize("passes", [1, 2])
@pytest.mark.parametrize("name", ["C2", "C5"])
def test_finalize_with_flatten_passes(h, name, passes):
    """ecl_cc_finalize with R23's passes first (ECL_CC_OPT_FLATTEN_PASSES) on unflattened
    local forests merged along the tree: same labels."""
    from paper_conf_hpdc_jaiganeshb18_b200 import dist
    g = gg.make_config(name, seed=11, scale_down=SMALL[name] + 1, device="cuda")
    expect, _ = oracle.bfs(*g.numpy())
    nindex64 = g.nindex.to(torch.int64)
    bounds = dist.partition_rows(nindex64, 4)
    forests = []
    for r in range(4):
        idx, lst = dist.slice_rows(nindex64, g.nlist, bounds[r], bounds[r + 1])
        forests.append(h.run_rows(g.n, bounds[r], bounds[r + 1], idx, lst, flatten=False))
    for (_, send, recv) in dist.tree_schedule(4):
        h.merge(forests[recv], forests[send])
    h.set_option("flatten_passes", passes)
    try:
        h.finalize(forests[0])
        torch.cuda.synchronize()
    finally:
        h.set_option("flatten_passes", 0)
    assert np.array_equal(forests[0].cpu().numpy(), expect)


def test_path_length_counters():
    """Table 4 analogue counters (stats build): every counted walk follows >= 1 pointer,
    the maximum bounds the average, and Jump3 (no compression) walks at least as far."""
    with ecl.Handle(0, stats=True) as hs:
        g = gg.make_config("C2", seed=1, scale_down=6, device="cuda")
        res = {}
        for jump in (4, 3):
            gpu_labels(hs, g, jump=jump)
            st = hs.stats()
            assert st["find_walks"] > 0 and st["path_len_max"] >= 1
            assert st["find_walks"] <= st["path_len_sum"] <= st["path_len_max"] * st["find_walks"]
            res[jump] = st["path_len_sum"] / st["find_walks"]
        assert res[3] >= res[4]


# ---------------------------------------------------------------------------------------
# R28 lazy Init3 (Init3 folded into the hook kernels): forced on and off everywhere
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("fuse", [0, 1, 2])
@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("seed", [1, 2])
def test_fuse_init_configs(h, name, fuse, seed):
    g = gg.make_config(name, seed=seed + 40, scale_down=SMALL[name], device="cuda")
    assert_parity(h, g, fuse_init=fuse)
    assert_parity(h, gg.shuffle_rows(g, seed=seed), fuse_init=fuse, order=0)


@pytest.mark.parametrize("g", hand_graphs(), ids=lambda g: g.name)
def test_fuse_init_hand_built(h, g):
    for fuse in (1, 2):
        assert_parity(h, g, fuse_init=fuse)
        assert_forest(h, g, fuse_init=fuse)


@pytest.mark.parametrize("opts", [dict(filter=1), dict(filter=0), dict(grid_blocks=3),
                                  dict(load_mode=0), dict(batch=0), dict(jump=2),
                                  dict(thresh_thread=4, thresh_warp=8), dict(order=1)],
                         ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
def test_fuse_init_options(h, opts):
    g = gg.make_config("C5", seed=3, scale_down=9, device="cuda")
    for fuse in (1, 2):
        assert_parity(h, g, fuse_init=fuse, **opts)
        assert_forest(h, gg.make_config("C4", seed=3, scale_down=8, device="cuda"),
                      fuse_init=fuse, **opts)


@pytest.mark.parametrize("G", [2, 4])
def test_fuse_init_multi_gpu(h, G):
    from paper_conf_hpdc_jaiganeshb18_b200 import dist
    g = gg.make_config("C5", seed=5, scale_down=10, device="cuda")
    expect, _ = oracle.bfs(*g.numpy())
    nindex64 = g.nindex.to(torch.int64)
    bounds = dist.partition_rows(nindex64, G)
    h.set_option("fuse_init", 1)
    try:
        forests = []
        for r in range(G):
            idx, lst = dist.slice_rows(nindex64, g.nlist, bounds[r], bounds[r + 1])
            forests.append(h.run_rows(g.n, bounds[r], bounds[r + 1], idx, lst, flatten=False))
        for (_, send, recv) in dist.tree_schedule(G):
            h.merge(forests[recv], forests[send])
        h.finalize(forests[0])
        torch.cuda.synchronize()
    finally:
        h.set_option("fuse_init", 2)
    assert np.array_equal(forests[0].cpu().numpy(), expect)


def test_fuse_init_auto_decision(h):
    """R28 auto: on for low-degree graphs with random vertex IDs (C1, C3), off for the
    mesh (C2: R23's passes shorten its Init3 chains) and for long rows (C4, C5: m >= 16n)."""
    want = {"C1": True, "C2": False, "C3": True, "C4": False, "C5": False}
    for name, lazy in want.items():
        g = gg.make_config(name, seed=1, scale_down=SMALL[name], device="cuda")
        assert_parity(h, g)
        info = h.run_info()
        assert info["lazy_init3"] == lazy, (name, info)


@pytest.mark.parametrize("G", [2, 4, 9])
@pytest.mark.parametrize("name", ["C4", "C5"])
@pytest.mark.parametrize("filt", [0, 1])
def test_fake_multi_gpu_encoded_merge_filter(name, G, filt):
    """dist.EncodedMerge's flow with one handle per fake rank: unflattened local forests
    (R21 filter forced on), peers encode with their own run's bitmap as membership proofs
    (ECL_CC_OPT_MERGE_FILTER), rank 0 merges into its own unflattened forest and flattens
    with its bitmap (extended by the merge)."""
    from paper_conf_hpdc_jaiganeshb18_b200 import dist
    g = gg.make_config(name, seed=17, scale_down=SMALL[name] + 1, device="cuda")
    expect, _ = oracle.bfs(*g.numpy())
    nindex64 = g.nindex.to(torch.int64)
    bounds = dist.partition_rows(nindex64, G, weights=dist.row_weights(nindex64, g.nlist))
    hs = [ecl.Handle(0) for _ in range(G)]
    try:
        forests, encs = [], []
        for r in range(G):
            hs[r].set_option("filter", 1).set_option("merge_filter", filt)
            idx, lst = dist.slice_rows(nindex64, g.nlist, bounds[r], bounds[r + 1])
            f = hs[r].run_rows(g.n, bounds[r], bounds[r + 1], idx, lst, flatten=False)
            forests.append(f)
            if r > 0:
                enc = hs[r].encode_buffers(g.n)
                hs[r].forest_encode(f, dist.row_anchor(idx, bounds[r]), enc)
                encs.append(enc)
        hs[0].merge_encoded(forests[0], encs)
        hs[0].finalize(forests[0])
        torch.cuda.synchronize()
        assert np.array_equal(forests[0].cpu().numpy(), expect)
    finally:
        for x in hs:
            x.close()

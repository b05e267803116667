"""Multi-process (gloo, CPU) tests of the multi-GPU driver's host logic (dist.py).

The transport (binomial tree of send/recv, chunked receives, broadcast) and the row
partitioning run for real over torch.distributed with the gloo backend on 127.0.0.1.
The per-rank compute is a CPU test double built on the oracle's union-find semantics —
test code may use the oracle; the product path never does.  The CUDA kernels behind the
same interface (run_rows / merge / finalize) are covered by tests/test_gpu_parity.py.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen as gg
import oracle
from paper_conf_hpdc_jaiganeshb18_b200 import dist as edist


def test_partition_rows_balanced_and_complete():
    g = gg.rmat(12, 8, seed=3)
    for world in (1, 2, 3, 4, 8):
        b = edist.partition_rows(g.nindex, world)
        assert b[0] == 0 and b[-1] == g.n and len(b) == world + 1
        assert all(b[i] <= b[i + 1] for i in range(world))
        nidx = g.nindex.to(torch.int64)
        per = [int(nidx[b[i + 1]] - nidx[b[i]]) for i in range(world)]
        assert sum(per) == g.m
        dmax = int(g.degrees().max())
        assert max(per) - g.m / world <= dmax + 1


def test_row_weights_count_probed_entries():
    """row_weights = 4 x #{u < v in row v} + 1 x deg(v) (STREAM_WEIGHT = 1/4), checked
    against a plain loop; the weighted partition balances those weights."""
    g = gg.rmat(10, 8, seed=5)
    nidx, nl = g.numpy()
    w = edist.row_weights(g.nindex, g.nlist, chunk=1000).numpy()
    for v in range(g.n):
        row = nl[nidx[v]:nidx[v + 1]]
        assert w[v] == 4 * int((row < v).sum()) + len(row)
    tw = torch.from_numpy(w)
    for world in (2, 3, 4, 8):
        b = edist.partition_rows(g.nindex, world, weights=tw)
        assert b[0] == 0 and b[-1] == g.n and all(b[i] <= b[i + 1] for i in range(world))
        per = [int(tw[b[i]:b[i + 1]].sum()) for i in range(world)]
        assert sum(per) == int(tw.sum())
        assert max(per) - int(tw.sum()) / world <= int(tw.max()) + 1


def test_tree_schedule_reaches_rank0():
    for world in range(1, 17):
        sched = edist.tree_schedule(world)
        alive = set(range(world))
        for (_, send, recv) in sched:
            assert send in alive and recv in alive and recv < send
            alive.discard(send)
        assert alive == {0}
        assert len(sched) == world - 1


class CpuOps:
    """Test double with the semantics of ecl_cc_run_rows / ecl_cc_merge / ecl_cc_finalize."""

    @staticmethod
    def _find(p, x):
        r = x
        while p[r] != r:
            r = p[r]
        while p[x] != r:
            p[x], x = r, p[x]
        return r

    def _union(self, p, a, b):
        ra, rb = self._find(p, a), self._find(p, b)
        if ra < rb:
            p[rb] = ra
        elif rb < ra:
            p[ra] = rb

    def run_rows(self, n, lo, hi, nindex_rows, nlist_rows):
        p = np.arange(n, dtype=np.int32)
        idx = nindex_rows.numpy()
        lst = nlist_rows.numpy()
        for r in range(hi - lo):
            v = lo + r
            for u in lst[idx[r]:idx[r + 1]]:
                if v > u:                                   # Fig. 6 line 1
                    self._union(p, v, int(u))
        for v in range(n):
            p[v] = self._find(p, v)
        return torch.from_numpy(p)

    def merge(self, parent, peer, v_lo):
        p = parent.numpy()
        pe = peer.numpy()
        for i in range(pe.shape[0]):
            if pe[i] != v_lo + i:
                self._union(p, v_lo + i, int(pe[i]))

    def finalize(self, parent):
        p = parent.numpy()
        for v in range(p.shape[0]):
            p[v] = self._find(p, v)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, seed, chunks, broadcast, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = gg.erdos_renyi(1500, 1400, seed=seed)       # many components
        ops = CpuOps()
        bounds = edist.partition_rows(g.nindex, world)
        lo, hi = bounds[rank], bounds[rank + 1]
        idx, lst = edist.slice_rows(g.nindex, g.nlist, lo, hi)
        parent = ops.run_rows(g.n, lo, hi, idx, lst)
        out = edist.forest_merge(parent, ops, chunks=chunks, broadcast=broadcast)
        q.put((rank, None if out is None else out.numpy().copy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,chunks,broadcast", [(2, 1, False), (2, 4, True), (3, 3, False),
                                                     (4, 2, True)])
def test_forest_merge_gloo(world, chunks, broadcast):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, 7, chunks, broadcast, q))
             for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    g = gg.erdos_renyi(1500, 1400, seed=7)
    expect, ncc = oracle.bfs(*g.numpy())
    assert ncc > 100
    assert np.array_equal(results[0], expect)
    for r in range(1, world):
        if broadcast:
            assert np.array_equal(results[r], expect)
        else:
            assert results[r] is None


def test_rebalance_weights_moves_rows_off_slow_ranks():
    """A rank measured twice as slow per weight unit gets fewer rows after rebalancing;
    equal measured times leave the partition (nearly) unchanged."""
    w = torch.ones(1000, dtype=torch.int64) * 4
    b = edist.partition_rows(torch.arange(1001), 4, weights=w)
    assert b == [0, 250, 500, 750, 1000]
    nb = edist.partition_rows(torch.arange(1001), 4,
                              weights=edist.rebalance_weights(w, b, [1.0, 1.0, 1.0, 2.0]))
    assert nb[0] == 0 and nb[-1] == 1000 and nb[4] - nb[3] < 250 and nb[1] > 250
    same = edist.partition_rows(torch.arange(1001), 4,
                                weights=edist.rebalance_weights(w, b, [3.0, 3.0, 3.0, 3.0]))
    assert all(abs(x - y) <= 1 for x, y in zip(same, b))

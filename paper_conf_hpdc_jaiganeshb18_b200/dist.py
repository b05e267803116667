"""Multi-GPU ECL-CC: row-partitioned local forests merged over NCCL.

Not in the paper (which is single-GPU); BASELINE.json's north_star adds it.  Each
rank owns a contiguous row range of the CSR chosen so every rank holds ~m/G entries.  It
builds a local forest of the edges stored in its rows with ``ecl_cc_run_rows`` (each
undirected edge (a,b), a > b, is hooked only by the owner of row a: Fig. 6 line 1), then
the forests are combined along a binomial tree: in round r the rank g with
g mod 2^(r+1) == 2^r sends its parent array to g - 2^r, which receives it in chunks and
hooks every (v, peer[v]) with ``ecl_cc_merge`` while the next chunk is in flight; only
rank 0's final forest is flattened (``ecl_cc_finalize``).  Rows are partitioned by
estimated work (``row_weights``: probed entries u < v plus a streaming share of all
entries), since the owner of high-ID rows probes most of its entries and the owner of
low-ID rows almost none.
Hook-once sufficiency makes the union of the forests' equivalence relations
exact, so rank 0 ends with the same min-ID labels as a single-GPU run.

The transport is a torch.distributed process group (NCCL on GPUs; gloo in the CPU tests);
the compute is whatever ``ops`` object is passed (the CUDA ``Handle`` in the product).
"""
from __future__ import annotations

from typing import List, Optional

import torch
import torch.distributed as dist


# Relative cost of an entry that is only streamed (u > v: Fig. 6 line 1 fails) against one
# that is also probed/hooked (u < v), from the measured probe-pattern ceiling
# (profiles/l2_ceiling.json: 2^30 entries streamed in ~0.66 ms, 2^29 probes ~1.38 ms more).
STREAM_WEIGHT = 0.25


def row_weights(nindex: torch.Tensor, nlist: torch.Tensor, chunk: int = 1 << 27) -> torch.Tensor:
    """Per-row work estimate for partitioning: entries with u < v (each probed and maybe
    hooked by the row's owner) + STREAM_WEIGHT x all entries (each streamed).  One pass
    over nlist on its device (setup, outside any timed region).  Returns int64 weights
    scaled by 4 (exact integers)."""
    nindex = nindex.to(torch.int64)
    n = nindex.numel() - 1
    m = int(nindex[-1])
    dev = nlist.device
    nidx = nindex.to(dev)
    lower = torch.zeros(n, dtype=torch.int64, device=dev)
    for a in range(0, m, chunk):
        pos = torch.arange(a, min(m, a + chunk), device=dev, dtype=torch.int64)
        rows = torch.searchsorted(nidx, pos, right=True) - 1
        lt = nlist[a:a + chunk].to(torch.int64) < rows
        lower.index_add_(0, rows[lt], torch.ones(int(lt.sum()), dtype=torch.int64, device=dev))
        del pos, rows, lt
    deg = nidx[1:] - nidx[:-1]
    return (4 * lower + int(4 * STREAM_WEIGHT) * deg).cpu()


def partition_rows(nindex: torch.Tensor, world: int,
                   weights: Optional[torch.Tensor] = None) -> List[int]:
    """Row bounds [b_0=0, ..., b_G=n] with ~1/G of the total weight per range: by default
    the directed entries (~m/G each), or per-row ``weights`` (e.g. ``row_weights``)."""
    nindex = nindex.to(torch.int64).cpu()
    n = nindex.numel() - 1
    if weights is not None:
        w = weights.to(torch.int64).cpu()
        nindex = torch.cat([torch.zeros(1, dtype=torch.int64), torch.cumsum(w, 0)])
    m = int(nindex[-1])
    targets = torch.tensor([(m * g) // world for g in range(1, world)], dtype=torch.int64)
    cuts = torch.searchsorted(nindex, targets, right=False).clamp_(0, n).tolist()
    bounds = [0] + cuts + [n]
    for i in range(1, len(bounds)):
        bounds[i] = max(bounds[i], bounds[i - 1])
    return bounds


def rebalance_weights(weights: torch.Tensor, bounds: List[int], rank_ms) -> torch.Tensor:
    """Per-row weights rescaled by each rank's MEASURED cost per weight unit (one untimed
    step of the current partition), for a second partition_rows call.  The static
    weights miss costs that depend on where the rows sit in the ID order: the owner of the
    highest IDs finds its rows' Init3 parents outside its range (identity roots)
    and does more hooking per probed entry."""
    w = weights.to(torch.float64).cpu().clone()
    for r in range(len(bounds) - 1):
        lo, hi = bounds[r], bounds[r + 1]
        tot = float(w[lo:hi].sum())
        if tot > 0 and rank_ms[r] > 0:
            w[lo:hi] *= float(rank_ms[r]) / tot
    total = float(w.sum())
    if total <= 0:
        return weights
    return (w * (2.0 ** 40 / total)).round().to(torch.int64)


def slice_rows(nindex: torch.Tensor, nlist: torch.Tensor, lo: int, hi: int):
    """CSR slice of rows [lo, hi): int64 offsets rebased to 0, and the adjacency view."""
    nindex = nindex.to(torch.int64)
    a = int(nindex[lo])
    b = int(nindex[hi])
    return (nindex[lo:hi + 1] - a).contiguous(), nlist[a:b]


def tree_schedule(world: int):
    """Binomial-tree rounds: list of (round, sender, receiver)."""
    out = []
    step = 1
    r = 0
    while step < world:
        for recv in range(0, world, 2 * step):
            send = recv + step
            if send < world:
                out.append((r, send, recv))
        step *= 2
        r += 1
    return out


def forest_merge(parent: torch.Tensor, ops, group=None, chunks: int = 4,
                 broadcast: bool = False) -> Optional[torch.Tensor]:
    """Combine every rank's forest ``parent`` (n entries, flattened or not) into rank 0's.

    Returns the global labels on rank 0 (and on every rank if ``broadcast``), else None.
    ``ops`` provides merge(parent, peer_chunk, v_lo) and finalize(parent).  With NCCL the
    device chunks go straight over NVLink; with gloo (CPU transport: the multi-process
    tests) device chunks are staged through host memory."""
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    n = parent.numel()
    staged = parent.is_cuda and dist.get_backend(group) == "gloo"
    bounds = [(n * c) // chunks for c in range(chunks + 1)]
    peer = None
    for (_, send, recv) in tree_schedule(world):
        if rank == send:
            for c in range(chunks):
                part = parent[bounds[c]:bounds[c + 1]]
                dist.send(part.cpu() if staged else part, dst=_g(group, recv), group=group)
            break
        if rank == recv:
            if peer is None:
                peer = torch.empty_like(parent)
                if staged:
                    host = torch.empty(n, dtype=parent.dtype, pin_memory=True)
            buf = host if staged else peer
            works = [dist.irecv(buf[bounds[c]:bounds[c + 1]], src=_g(group, send), group=group)
                     for c in range(chunks)]
            for c in range(chunks):
                works[c].wait()  # orders the compute stream after chunk c only
                if staged:
                    peer[bounds[c]:bounds[c + 1]].copy_(host[bounds[c]:bounds[c + 1]])
                ops.merge(parent, peer[bounds[c]:bounds[c + 1]], bounds[c])
            if staged:
                torch.cuda.current_stream(parent.device).synchronize()  # host buffer reuse
    # Only rank 0's final forest is flattened: a forest that is sent on or merged again
    # needs no flattening, since (v, parent[v]) for every v spans the same trees as
    # (v, root(v)) (hook-once sufficiency).
    if rank == 0:
        ops.finalize(parent)
    if broadcast:
        if staged:
            host = parent.cpu()
            dist.broadcast(host, src=_g(group, 0), group=group)
            parent.copy_(host)
        else:
            dist.broadcast(parent, src=_g(group, 0), group=group)
        return parent
    return parent if rank == 0 else None


def row_anchor(nindex_rows: torch.Tensor, lo: int) -> int:
    """The highest-degree row of a slice (the encoding's anchor: its label is normally the
    rank's giant component, so the bitmap holds most vertices and the pair list is
    short)."""
    deg = (nindex_rows[1:] - nindex_rows[:-1]).to(torch.int64)
    return lo + int(torch.argmax(deg)) if deg.numel() else -1     # -1: empty slice


class EncodedMerge:
    """Flat merge of encoded forests into rank 0 (the variants the survey
    lists beside the binomial tree of full forests).

    Every rank g != 0 encodes its (unflattened) local forest (ecl_cc_forest_encode: an
    n/32-word bitmap of "root == D" plus the pairs (v, root(v)) of the remaining non-roots
    — for a power-law graph 16 MB + a few MB instead of the 537 MB parent array at
    n = 2^27), and rank 0 hooks all peers' relations into its own local forest in one
    ecl_cc_merge_encoded call, then flattens once.  With ECL_CC_OPT_MERGE_FILTER every
    step uses the R21 anchor bitmap of the rank's own local run as membership proofs, so
    most vertices of the giant tree need no random walk (the walks of a local forest's
    flatten are random DRAM reads at n = 2^27).  Exact by hook-once sufficiency
    (P:L161-L163): the encoded edges span the same classes as the labels.

    mode "compact": the encodings travel over the process group (NCCL send/recv; gloo
      stages through host memory).  The pair count is exchanged first (one small host
      synchronisation per step) so only the used part of the pair buffer is sent.
    mode "p2p": no copies.  Each rank exports its encoding buffers once (CUDA IPC,
      ecl_cc_ipc_export); rank 0 maps them (ecl_cc_ipc_open) and its merge kernels read
      the peers' bitmaps and pairs directly over NVLink, so the transfer happens inside the
      merge.  The process group only orders the steps: a one-int "encoded" signal from
      every peer before the merge and an "done reading" acknowledgement back after it.
      With NCCL both are stream-ordered device operations (no host synchronisation); with
      gloo (tests, one GPU) the streams are synchronised around host messages.
    """

    # handle options around the merge's calls (restored afterwards)
    OPTS = {"merge_filter": 1}

    def __init__(self, handle, n: int, anchor: int, mode: str = "p2p", group=None,
                 opts: Optional[dict] = None):
        if mode not in ("compact", "p2p"):
            raise ValueError(mode)
        self.h, self.n, self.anchor, self.mode, self.group = handle, n, anchor, mode, group
        self.opts = dict(self.OPTS if opts is None else opts)
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        if self.world - 1 > 8:
            raise ValueError("EncodedMerge merges at most 8 peers into rank 0")
        self.gloo = dist.get_backend(group) == "gloo"
        dev = handle.device
        self.flag = torch.ones(1, dtype=torch.int32, device=dev)
        self.enc = handle.encode_buffers(n) if self.rank != 0 else None
        self.peers = []
        self.mapped = []
        if mode == "p2p":
            hs = None
            if self.rank != 0:
                hs = {k: handle.ipc_export(self.enc[k]) for k in ("bits", "pairs", "meta")}
            allh = [None] * self.world
            dist.all_gather_object(allh, hs, group=group)
            if self.rank == 0:
                for r in range(1, self.world):
                    ptrs = {k: handle.ipc_open(allh[r][k]) for k in ("bits", "pairs", "meta")}
                    self.mapped += list(ptrs.values())
                    self.peers.append({**ptrs, "cap": n})
        elif self.rank == 0:
            self.recv = [handle.encode_buffers(n) for _ in range(1, self.world)]

    def _with_opts(self, fn, *a):
        for k, v in self.opts.items():
            self.h.set_option(k, v)
        try:
            return fn(*a)
        finally:
            for k in self.opts:
                self.h.set_option(k, 0)

    def close(self):
        for p in self.mapped:
            self.h.ipc_close(p)
        self.mapped = []

    # -- transport helpers (NCCL: stream-ordered device ops; gloo: host messages) --------
    def _send(self, t, dst):
        if self.gloo and t.is_cuda:
            t = t.cpu()                       # synchronises the stream first
        dist.send(t, dst=_g(self.group, dst), group=self.group)

    def _recv(self, t, src):
        if self.gloo and t.is_cuda:
            host = torch.empty(t.shape, dtype=t.dtype)
            dist.recv(host, src=_g(self.group, src), group=self.group)
            t.copy_(host)
        else:
            dist.recv(t, src=_g(self.group, src), group=self.group)

    def __call__(self, parent: torch.Tensor, broadcast: bool = False):
        h, rank = self.h, self.rank
        if self.world == 1:
            self._with_opts(h.finalize, parent)
        elif rank != 0:
            self._with_opts(h.forest_encode, parent, self.anchor, self.enc)
            if self.mode == "p2p":
                self._send(self.flag, 0)                    # "my encoding is complete"
                self._recv(self.flag, 0)                    # rank 0 finished reading it
            else:
                meta = self.enc["meta"]
                self._send(meta, 0)
                npairs = int(meta[0].item())
                self._send(self.enc["bits"], 0)
                if npairs:
                    self._send(self.enc["pairs"][:2 * npairs], 0)
        else:
            if self.mode == "p2p":
                for r in range(1, self.world):
                    self._recv(self.flag, r)
                self._with_opts(h.merge_encoded, parent, self.peers)
                if self.gloo:
                    torch.cuda.current_stream(parent.device).synchronize()
                for r in range(1, self.world):
                    self._send(self.flag, r)
            else:
                peers = []
                for r, buf in zip(range(1, self.world), self.recv):
                    self._recv(buf["meta"], r)
                    npairs = int(buf["meta"][0].item())
                    self._recv(buf["bits"], r)
                    if npairs:
                        self._recv(buf["pairs"][:2 * npairs], r)
                    peers.append({"bits": buf["bits"], "pairs": buf["pairs"],
                                  "meta": buf["meta"], "cap": npairs})
                self._with_opts(h.merge_encoded, parent, peers)
            self._with_opts(h.finalize, parent)
        if broadcast:
            if self.gloo and parent.is_cuda:
                host = parent.cpu()
                dist.broadcast(host, src=_g(self.group, 0), group=self.group)
                parent.copy_(host)
            else:
                dist.broadcast(parent, src=_g(self.group, 0), group=self.group)
            return parent
        return parent if rank == 0 else None


def _g(group, r):
    return r if group is None else dist.get_global_rank(group, r)


def run_distributed(nindex: torch.Tensor, nlist: torch.Tensor, handle, group=None,
                    chunks: int = 4, broadcast: bool = False, bounds=None):
    """Whole-graph CSR visible on every rank (device tensors); each rank processes its row
    range, then the forests are merged.  Returns labels on rank 0 (all ranks if
    ``broadcast``)."""
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    n = nindex.numel() - 1
    if bounds is None:
        bounds = partition_rows(nindex, world)
    lo, hi = bounds[rank], bounds[rank + 1]
    idx, lst = slice_rows(nindex, nlist, lo, hi)
    parent = handle.run_rows(n, lo, hi, idx, lst, flatten=False)
    return forest_merge(parent, handle, group=group, chunks=chunks, broadcast=broadcast)

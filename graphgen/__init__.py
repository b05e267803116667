"""Seeded synthetic graph generators shaped like the paper's inputs (Table 2).

This module is shared by both sides of the parity tests (the CPU oracle and the CUDA path)
and holds NONE of the method's arithmetic: it only produces CSR graphs.  It is written with
integer-only torch tensor ops so the same seed gives bit-identical graphs on CPU and on
CUDA (the GPU is used only to make the large configs fast to build).

Randomness: a counter-based splitmix64 hash ``h(seed, stream, i)`` (no RNG state), so any
element can be recomputed independently.  A uniform vertex in [0, n) is
``((h >>> 32) * n) >>> 32``; Bernoulli(p) is ``(h >>> 32) < floor(p * 2^32)``.

CSR convention (§4): self-loops and multi-edges removed, every undirected edge
stored as two directed entries, rows sorted ascending by neighbour ID.

Configs (BASELINE.json ``configs``; readings pinned in SURVEY §4 and DESIGN.md §3):
  C1  Erdos-Renyi G(n, M), n = 2^16, M = 2n uniform pairs            (avg degree 4)
  C2  4096 x 4096 4-neighbour grid, row-major IDs, 10 % edges deleted
  C3  "r4-2e23": every vertex draws 4 uniform targets, n = 2^23
  C4  R-MAT scale 24, edge factor 16, (a,b,c,d) = (.55,.10,.10,.25), no permutation
  C5  Graph500 Kronecker scale 27, edge factor 16, (.57,.19,.19,.05), random permutation
"""
from __future__ import annotations

import dataclasses
from typing import Optional

import torch

_MASK32 = (1 << 32) - 1


def _s64(x: int) -> int:
    """Python int in [0, 2^64) -> the int64 with the same bits."""
    x &= (1 << 64) - 1
    return x - (1 << 64) if x >= (1 << 63) else x


_GOLDEN = _s64(0x9E3779B97F4A7C15)
_M1 = _s64(0xBF58476D1CE4E5B9)
_M2 = _s64(0x94D049BB133111EB)
_STREAM = _s64(0xD1B54A32D192ED03)


def _shr(z: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (z >> k) & ((1 << (64 - k)) - 1)


def mix64(z: torch.Tensor) -> torch.Tensor:
    """splitmix64 finaliser on int64 tensors (two's-complement wrap-around arithmetic)."""
    z = (z ^ _shr(z, 30)) * _M1
    z = (z ^ _shr(z, 27)) * _M2
    return z ^ _shr(z, 31)


def hash64(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """h(seed, stream, i): independent 64-bit words for every counter value i."""
    base = _s64(mix64(torch.tensor([_s64(seed * 0x9E3779B97F4A7C15 + stream * 0xD1B54A32D192ED03)],
                                   dtype=torch.int64)).item())
    return mix64(idx.to(torch.int64) * _GOLDEN + base)


def hash64_ref(seed: int, stream: int, i: int) -> int:
    """Pure-Python reference of ``hash64`` (unsigned result), for tests."""
    M = (1 << 64) - 1

    def mix(z):
        z &= M
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
        return z ^ (z >> 31)

    base = mix(seed * 0x9E3779B97F4A7C15 + stream * 0xD1B54A32D192ED03)
    return mix(i * 0x9E3779B97F4A7C15 + base)


def hi32(h: torch.Tensor) -> torch.Tensor:
    return _shr(h, 32)


def lo32(h: torch.Tensor) -> torch.Tensor:
    return h & _MASK32


def uniform_vertex(w32: torch.Tensor, n: int) -> torch.Tensor:
    """Map a 32-bit random word to [0, n) by multiply-shift (no modulo bias issues)."""
    return (w32 * n) >> 32


# ----------------------------------------------------------------------------------------
# CSR assembly
# ----------------------------------------------------------------------------------------
@dataclasses.dataclass
class Graph:
    """Undirected graph in CSR.  ``nindex`` has n+1 offsets (int32 if m < 2^31 else int64),
    ``nlist`` holds m int32 neighbour IDs.  Tensors live on the device they were built on."""
    name: str
    n: int
    nindex: torch.Tensor
    nlist: torch.Tensor

    @property
    def m(self) -> int:
        return int(self.nlist.numel())

    def to(self, device) -> "Graph":
        return Graph(self.name, self.n, self.nindex.to(device), self.nlist.to(device))

    def numpy(self):
        return self.nindex.cpu().numpy(), self.nlist.cpu().numpy()

    def degrees(self) -> torch.Tensor:
        return (self.nindex[1:] - self.nindex[:-1]).to(torch.int64)


def csr_from_pairs(name: str, n: int, src: torch.Tensor, dst: torch.Tensor,
                   index_dtype: Optional[torch.dtype] = None, buckets: int = 1) -> Graph:
    """Symmetrize, drop self-loops, sort by (row, col), dedupe, build offsets.

    ``buckets`` > 1 splits the work by source-row range so that no single sort exceeds
    ~1/buckets of the directed entries (needed for the 4e9-entry Kronecker config); the
    endpoint arrays stay in their input dtype and only one bucket's int64 keys exist at a
    time."""
    device = src.device
    if src.dtype not in (torch.int32, torch.int64):
        src = src.to(torch.int64)
    if dst.dtype != src.dtype:
        dst = dst.to(src.dtype)
    counts = torch.zeros(n, dtype=torch.int64, device=device)
    cols = []
    bounds = [(n * b) // buckets for b in range(buckets + 1)]
    for b in range(buckets):
        lo, hi = bounds[b], bounds[b + 1]
        parts = []
        for a, c in ((src, dst), (dst, src)):
            sel = (a >= lo) & (a < hi) & (a != c)
            aa = a[sel].to(torch.int64)
            cc = c[sel].to(torch.int64)
            del sel
            parts.append((aa - lo) * n + cc)
            del aa, cc
        keys = torch.unique(torch.cat(parts), sorted=True)
        del parts
        rows = keys // n
        counts[lo:hi] = torch.bincount(rows, minlength=hi - lo)
        cols.append((keys - rows * n).to(torch.int32))
        del keys, rows
    nlist = torch.cat(cols) if len(cols) > 1 else (
        cols[0] if cols else torch.zeros(0, dtype=torch.int32, device=device))
    del cols
    m = nlist.numel()
    if index_dtype is None:
        index_dtype = torch.int32 if m < 2 ** 31 else torch.int64
    nindex = torch.zeros(n + 1, dtype=torch.int64, device=device)
    torch.cumsum(counts, 0, out=nindex[1:])
    return Graph(name, n, nindex.to(index_dtype), nlist)


def from_edges(n: int, edges, name: str = "edges", index_dtype=None) -> Graph:
    """Small hand-built graphs: ``edges`` is an iterable of undirected (a, b) pairs."""
    e = torch.tensor(list(edges), dtype=torch.int64).reshape(-1, 2)
    return csr_from_pairs(name, n, e[:, 0], e[:, 1], index_dtype=index_dtype)


# ----------------------------------------------------------------------------------------
# Generators
# ----------------------------------------------------------------------------------------
def erdos_renyi(n: int, M: int, seed: int = 1, device="cpu") -> Graph:
    """G(n, M): M uniform (u, v) pairs (C1 reading)."""
    i = torch.arange(M, dtype=torch.int64, device=device)
    src = uniform_vertex(hi32(hash64(seed, 0, i)), n)
    dst = uniform_vertex(hi32(hash64(seed, 1, i)), n)
    return csr_from_pairs(f"er_n{n}_M{M}_s{seed}", n, src, dst)


def grid2d(rows: int, cols: int, p_delete: float = 0.0, seed: int = 1, device="cpu") -> Graph:
    """4-neighbour grid with row-major IDs v = r*cols + c; each undirected edge is deleted
    independently with probability p_delete (C2; p=0 gives Table 2's 2d-2e20.sym)."""
    thr = int(p_delete * (1 << 32))
    r = torch.arange(rows, dtype=torch.int64, device=device)
    c = torch.arange(cols, dtype=torch.int64, device=device)
    # horizontal edges (r,c)-(r,c+1), counter e = r*(cols-1)+c
    hs = (r[:, None] * cols + c[None, :-1]).reshape(-1)
    he = (r[:, None] * (cols - 1) + c[None, :-1]).reshape(-1)
    # vertical edges (r,c)-(r+1,c), counter e = r*cols+c
    vs = (r[:-1, None] * cols + c[None, :]).reshape(-1)
    ve = vs.clone()
    keep_h = hi32(hash64(seed, 0, he)) >= thr
    keep_v = hi32(hash64(seed, 1, ve)) >= thr
    src = torch.cat([hs[keep_h], vs[keep_v]])
    dst = torch.cat([hs[keep_h] + 1, vs[keep_v] + cols])
    n = rows * cols
    return csr_from_pairs(f"grid{rows}x{cols}_del{p_delete}_s{seed}", n, src, dst)


def random_kout(n: int, k: int = 4, seed: int = 1, device="cpu") -> Graph:
    """k-out random graph: each vertex draws k uniform targets (Galois "r4" reading, C3)."""
    v = torch.arange(n, dtype=torch.int64, device=device)
    src = v.repeat(k)
    dst = torch.cat([uniform_vertex(hi32(hash64(seed, j, v)), n) for j in range(k)])
    return csr_from_pairs(f"r{k}_n{n}_s{seed}", n, src, dst)


def _rmat_pairs(scale: int, nsamples: int, a: float, b: float, c: float, seed: int,
                first: int, device) -> tuple:
    """R-MAT quadrant recursion for samples [first, first+nsamples): at every level a
    32-bit word picks quadrant (0,0) w.p. a, (0,1) w.p. b, (1,0) w.p. c, (1,1) otherwise."""
    ta = int(a * (1 << 32))
    tab = int((a + b) * (1 << 32))
    tabc = int((a + b + c) * (1 << 32))
    i = torch.arange(first, first + nsamples, dtype=torch.int64, device=device)
    row = torch.zeros_like(i)
    col = torch.zeros_like(i)
    for lvl in range(scale):
        h = hash64(seed, 1000 + lvl // 2, i)
        w = hi32(h) if lvl % 2 == 0 else lo32(h)
        bit = 1 << (scale - 1 - lvl)
        right = ((w >= ta) & (w < tab)) | (w >= tabc)
        down = w >= tab
        row |= down.to(torch.int64) * bit
        col |= right.to(torch.int64) * bit
        del h, w
    return row, col


def vertex_permutation(n: int, seed: int, device="cpu") -> torch.Tensor:
    """Deterministic random permutation of [0, n): sort by (hash, index) keys.  Gives the
    same permutation on every device (unlike torch.randperm)."""
    idx = torch.arange(n, dtype=torch.int64, device=device)
    bits = max(1, (n - 1).bit_length())
    key = (hi32(hash64(seed, 7777, idx)) << bits) | idx  # unique by construction
    return torch.argsort(key)


def rmat(scale: int, edge_factor: int, abc=(0.55, 0.10, 0.10), seed: int = 1,
         permute: bool = False, device="cpu", chunk: int = 1 << 27, buckets: int = 1) -> Graph:
    """R-MAT / Kronecker edge list of edge_factor * 2^scale undirected samples."""
    n = 1 << scale
    total = edge_factor * n
    srcs, dsts = [], []
    for first in range(0, total, chunk):
        r, c = _rmat_pairs(scale, min(chunk, total - first), *abc, seed=seed, first=first,
                           device=device)
        srcs.append(r.to(torch.int32))
        dsts.append(c.to(torch.int32))
        del r, c
    src = torch.cat(srcs)
    del srcs
    dst = torch.cat(dsts)
    del dsts
    if permute:
        perm = vertex_permutation(n, seed, device).to(torch.int32)
        src = perm[src.long()]
        dst = perm[dst.long()]
        del perm
    name = ("kron" if permute else "rmat") + f"_s{scale}_ef{edge_factor}_seed{seed}"
    return csr_from_pairs(name, n, src, dst, buckets=buckets)


def graph500(scale: int, edge_factor: int = 16, seed: int = 1, device="cpu", **kw) -> Graph:
    """Graph500 Kronecker generator parameters (0.57, 0.19, 0.19, 0.05) + vertex permutation."""
    return rmat(scale, edge_factor, (0.57, 0.19, 0.19), seed=seed, permute=True,
                device=device, **kw)


# ----------------------------------------------------------------------------------------
# BASELINE.json configs
# ----------------------------------------------------------------------------------------
CONFIGS = {
    "C1": "uniform random graph n=2^16, avg degree 4 (Erdos-Renyi G(n, M=2n))",
    "C2": "2D grid 4096x4096 with 10% random edge deletions",
    "C3": "uniform random r4-2^23 (4-out random graph)",
    "C4": "R-MAT scale 24 edge factor 16 (0.55,0.10,0.10,0.25)",
    "C5": "Kronecker/Graph500 scale 27 edge factor 16 (0.57,0.19,0.19,0.05), permuted",
}


def make_config(name: str, seed: int = 1, device="cpu", scale_down: int = 0) -> Graph:
    """Build config C1..C5.  ``scale_down`` shrinks the graph (by 2^scale_down vertices)
    with the same recipe, for CPU-sized parity cases."""
    s = scale_down
    if name == "C1":
        n = 1 << (16 - s)
        return erdos_renyi(n, 2 * n, seed=seed, device=device)
    if name == "C2":
        side = 4096 >> ((s + 1) // 2)
        return grid2d(side, side, 0.10, seed=seed, device=device)
    if name == "C3":
        return random_kout(1 << (23 - s), 4, seed=seed, device=device)
    if name == "C4":
        return rmat(24 - s, 16, (0.55, 0.10, 0.10), seed=seed, device=device,
                    buckets=1 if s > 0 else 2)
    if name == "C5":
        return graph500(27 - s, 16, seed=seed, device=device,
                        buckets=1 if s > 3 else 16, chunk=1 << 27)
    raise KeyError(name)


def raw_csr(name: str, n: int, rows: torch.Tensor, cols: torch.Tensor,
            seed: Optional[int] = None, index_dtype: Optional[torch.dtype] = None) -> Graph:
    """CSR of the directed entries (rows[i], cols[i]) exactly as given — no symmetrising,
    no loop removal, no dedupe — with every row's entries in a seeded random order, or in
    their given order when ``seed`` is None."""
    rows = rows.to(torch.int64)
    cols = cols.to(torch.int64)
    device = rows.device
    E = rows.numel()
    i = torch.arange(E, dtype=torch.int64, device=device)
    key = (rows << 32) | (i if seed is None else hi32(hash64(seed, 4343, i)))
    order = torch.argsort(key)
    nlist = cols[order].to(torch.int32).contiguous()
    nindex = torch.zeros(n + 1, dtype=torch.int64, device=device)
    if E:
        torch.cumsum(torch.bincount(rows, minlength=n), 0, out=nindex[1:])
    if index_dtype is None:
        index_dtype = torch.int32 if E < 2 ** 31 else torch.int64
    return Graph(name, n, nindex.to(index_dtype), nlist)


def inject_loops_dups(g: Graph, seed: int, p_loop: float = 0.1, p_dup: float = 0.1) -> Graph:
    """A raw CSR with the same components as ``g`` (whose entries are kept): a self-loop
    (v, v) added to each vertex with probability p_loop, each directed entry (a, b)
    duplicated with probability p_dup together with a copy of (b, a) (so the input stays
    symmetric), and every row's entries shuffled, so loops and duplicates land anywhere in
    a row (also among the first entries Init3 reads).  SURVEY §8(b) "accepted inputs"."""
    device = g.nlist.device
    deg = g.degrees()
    rows = torch.repeat_interleave(torch.arange(g.n, dtype=torch.int64, device=device), deg)
    cols = g.nlist.to(torch.int64)
    v = torch.arange(g.n, dtype=torch.int64, device=device)
    loop = v[hi32(hash64(seed, 4444, v)) < int(p_loop * (1 << 32))]
    e = torch.arange(g.m, dtype=torch.int64, device=device)
    dup = e[hi32(hash64(seed, 4545, e)) < int(p_dup * (1 << 32))]
    R = torch.cat([rows, loop, rows[dup], cols[dup]])
    C = torch.cat([cols, loop, cols[dup], rows[dup]])
    return raw_csr(g.name + f"_loopdup{seed}", g.n, R, C, seed,
                   index_dtype=g.nindex.dtype)


def shuffle_rows(g: Graph, seed: int) -> Graph:
    """Randomly permute the entries inside every row (reading R4: order-independence)."""
    deg = g.degrees()
    rows = torch.repeat_interleave(torch.arange(g.n, dtype=torch.int64, device=g.nlist.device), deg)
    key = (rows << 32) | hi32(hash64(seed, 4242, torch.arange(g.m, dtype=torch.int64,
                                                               device=g.nlist.device)))
    order = torch.argsort(key)
    return Graph(g.name + f"_shuf{seed}", g.n, g.nindex.clone(), g.nlist[order].contiguous())

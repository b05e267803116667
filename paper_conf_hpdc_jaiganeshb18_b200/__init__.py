"""B200-native ECL-CC connected components (Jaiganesh & Burtscher, HPDC '18).

Thin Python binding over the C ABI of ``libecl_cc.so`` (declared in ``include/ecl_cc.h``).
This module only marshals arguments: it checks dtypes/devices, passes raw pointers and the
current CUDA stream, and raises on error.  Every step of the method runs in the library's
CUDA kernels; there is no CPU or PyTorch fallback — if the library is missing, importing
the binding works but every call raises ``RuntimeError`` (run ``__graft_entry__.build()``).

Typical use::

    import torch, paper_conf_hpdc_jaiganeshb18_b200 as ecl
    labels = ecl.run(nindex, nlist)          # CUDA tensors; labels[v] = min ID of v's CC

PAPER.md references: problem statement P:L45 (§1); method P:L135-L181 (§3).
"""
from __future__ import annotations

import ctypes
import os
import threading
from typing import Optional

import torch

from . import build as _build

__all__ = ["Handle", "run", "run_host", "EclCCError", "library_path", "OPT", "read_mtx",
           "read_edgelist"]

OPT = {
    "thresh_thread": 1,
    "thresh_warp": 2,
    "grid_blocks": 3,
    "stop_after": 4,
    "load_mode": 5,
    "timing": 6,
    "ttas": 7,
    "l2_fetch": 8,
    "occ_thread": 9,
    "occ_range": 10,
    "init": 11,
    "jump": 12,
    "fini": 13,
    "batch": 14,
    "filter": 15,
    "order": 16,
    "prejump": 17,
    "flatten_passes": 18,
    "fuse_init": 19,
    "merge_filter": 20,
    "vec": 21,
    "fused": 22,
}
PHASES = ("init_bin", "hook_thread", "hook_warp", "hook_block", "finalize")

_STATUS = {0: "ok", 1: "invalid argument", 2: "CUDA error", 3: "out of device memory",
           4: "invalid graph"}


class EclCCError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"ecl_cc: {_STATUS.get(status, status)}: {msg}")
        self.status = status


_libs = {}
_lock = threading.Lock()


def library_path(stats: bool = False) -> str:
    if not stats and os.environ.get("ECL_CC_LIB"):   # dev A/B builds (tools/ab.sh)
        return os.environ["ECL_CC_LIB"]
    return _build.lib_path("libecl_cc_stats.so" if stats else "libecl_cc.so")


def _load(stats: bool = False) -> ctypes.CDLL:
    with _lock:
        if stats in _libs:
            return _libs[stats]
        path = library_path(stats)
        if not os.path.exists(path):
            raise RuntimeError(f"CUDA library {path} is not built; run "
                               "`python -c 'import __graft_entry__ as g; g.build()'`")
        lib = ctypes.CDLL(path)
        P, I32, I64, INT = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_int
        sig = {
            "ecl_cc_create": ([ctypes.POINTER(P), INT], INT),
            "ecl_cc_destroy": ([P], INT),
            "ecl_cc_run": ([P, I32, I64, P, P, P, P], INT),
            "ecl_cc_run_i64": ([P, I32, I64, P, P, P, P], INT),
            "ecl_cc_run_host": ([P, I32, I64, P, INT, P, P, P], INT),
            "ecl_cc_spanning_forest": ([P, I32, I64, P, INT, P, P, P, P, P], INT),
            "ecl_cc_run_rows": ([P, I32, I32, I32, I64, P, P, P, P], INT),
            "ecl_cc_build_csr": ([P, I32, I64, P, P, P, P, I64, ctypes.POINTER(I64), P], INT),
            "ecl_cc_read_mtx": ([ctypes.c_char_p, ctypes.POINTER(I32), ctypes.POINTER(I64),
                                 ctypes.POINTER(P), ctypes.POINTER(P)], INT),
            "ecl_cc_read_edgelist": ([ctypes.c_char_p, ctypes.POINTER(I32), ctypes.POINTER(I64),
                                      ctypes.POINTER(P), ctypes.POINTER(P)], INT),
            "ecl_cc_free_host": ([P], None),
            "ecl_cc_io_last_error": ([], ctypes.c_char_p),
            "ecl_cc_merge": ([P, I32, I32, I32, P, P, P], INT),
            "ecl_cc_finalize": ([P, I32, P, P], INT),
            "ecl_cc_forest_encode": ([P, I32, P, I32, P, P, I64, P, P], INT),
            "ecl_cc_merge_encoded": ([P, I32, INT, ctypes.POINTER(P), ctypes.POINTER(P),
                                      ctypes.POINTER(P), ctypes.POINTER(I64), P, P], INT),
            "ecl_cc_ipc_export": ([P, P], INT),
            "ecl_cc_ipc_open": ([INT, P, ctypes.POINTER(P)], INT),
            "ecl_cc_ipc_close": ([P], INT),
            "ecl_cc_validate": ([P, I32, I64, P, INT, P, P], INT),
            "ecl_cc_set_option": ([P, INT, I64], INT),
            "ecl_cc_get_worklist": ([P, P, ctypes.POINTER(I64), P, ctypes.POINTER(I64)], INT),
            "ecl_cc_get_stats": ([P, ctypes.POINTER(I64)], INT),
            "ecl_cc_get_stats_ex": ([P, ctypes.POINTER(I64), INT], INT),
            "ecl_cc_get_run_info": ([P, ctypes.POINTER(I64), INT], INT),
            "ecl_cc_get_filter": ([P, ctypes.POINTER(P), ctypes.POINTER(I64),
                                   ctypes.POINTER(I32)], INT),
            "ecl_cc_stats_enabled": ([], INT),
            "ecl_cc_get_timing": ([P, ctypes.POINTER(ctypes.c_float)], INT),
            "ecl_cc_status_string": ([INT], ctypes.c_char_p),
            "ecl_cc_last_error": ([P], ctypes.c_char_p),
            "ecl_cc_version": ([], ctypes.c_char_p),
        }
        for name, (args, res) in sig.items():
            f = getattr(lib, name)
            f.argtypes = args
            f.restype = res
        _libs[stats] = lib
        return lib


IPC_HANDLE_BYTES = 72   # ECL_CC_IPC_HANDLE_BYTES


def _addr(x) -> int:
    """A device address: a tensor's data pointer or a raw int (e.g. an IPC mapping)."""
    return x.data_ptr() if isinstance(x, torch.Tensor) else int(x)


def _ptr(t: Optional[torch.Tensor]):
    return ctypes.c_void_p(t.data_ptr()) if t is not None and t.numel() > 0 else ctypes.c_void_p(0)


def _stream_ptr(stream, device) -> ctypes.c_void_p:
    if stream is None:
        stream = torch.cuda.current_stream(device)
    if isinstance(stream, torch.cuda.Stream):
        return ctypes.c_void_p(stream.cuda_stream)
    return ctypes.c_void_p(int(stream))


def _dev_tensor(t: torch.Tensor, name: str, dtypes, device: torch.device):
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch tensor")
    if t.dtype not in dtypes:
        raise TypeError(f"{name} must have dtype in {dtypes}, got {t.dtype}")
    if t.device != device:
        raise ValueError(f"{name} must live on {device}, got {t.device}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return t


class Handle:
    """Owns an ``ecl_cc_handle`` (device scratch + options) bound to one CUDA device."""

    def __init__(self, device=None, stats: bool = False):
        if not torch.cuda.is_available():
            raise RuntimeError("ecl_cc needs a CUDA device (no CPU fallback exists)")
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None
                                   else torch.device(device).index or 0)
        self._lib = _load(stats)
        h = ctypes.c_void_p()
        st = self._lib.ecl_cc_create(ctypes.byref(h), self.device.index)
        if st != 0:
            raise EclCCError(st, "ecl_cc_create failed")
        self._h = h

    # -- plumbing ---------------------------------------------------------------------
    def _check(self, st: int):
        if st != 0:
            raise EclCCError(st, self._lib.ecl_cc_last_error(self._h).decode())

    def close(self):
        if getattr(self, "_h", None):
            self._lib.ecl_cc_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    @property
    def stats_enabled(self) -> bool:
        return bool(self._lib.ecl_cc_stats_enabled())

    def set_option(self, name: str, value: int) -> "Handle":
        self._check(self._lib.ecl_cc_set_option(self._h, OPT[name], int(value)))
        return self

    # -- the operation ----------------------------------------------------------------
    def run(self, nindex: torch.Tensor, nlist: torch.Tensor, out: Optional[torch.Tensor] = None,
            stream=None) -> torch.Tensor:
        """labels[v] = min vertex ID of v's component (enqueued on ``stream``)."""
        d = self.device
        _dev_tensor(nindex, "nindex", (torch.int32, torch.int64), d)
        _dev_tensor(nlist, "nlist", (torch.int32,), d)
        n = nindex.numel() - 1
        if n < 0:
            raise ValueError("nindex must hold n+1 offsets")
        if out is None:
            out = torch.empty(n, dtype=torch.int32, device=d)
        _dev_tensor(out, "out", (torch.int32,), d)
        if out.numel() != n:
            raise ValueError("out must have n entries")
        m = nlist.numel()
        fn = self._lib.ecl_cc_run if nindex.dtype == torch.int32 else self._lib.ecl_cc_run_i64
        self._check(fn(self._h, n, m, _ptr(nindex), _ptr(nlist), _ptr(out),
                       _stream_ptr(stream, d)))
        return out

    def spanning_forest(self, nindex: torch.Tensor, nlist: torch.Tensor, stream=None):
        """(labels, tree_a, tree_b): min-ID labels and, for every vertex x that is not its
        component's minimum, a CSR edge (tree_a[x], tree_b[x]); together these edges form a
        spanning forest (ecl_cc_spanning_forest).  Entries of component minima are -1."""
        d = self.device
        _dev_tensor(nindex, "nindex", (torch.int32, torch.int64), d)
        _dev_tensor(nlist, "nlist", (torch.int32,), d)
        n = nindex.numel() - 1
        if n < 0:
            raise ValueError("nindex must hold n+1 offsets")
        labels = torch.empty(n, dtype=torch.int32, device=d)
        ta = torch.empty(n, dtype=torch.int32, device=d)
        tb = torch.empty(n, dtype=torch.int32, device=d)
        self._check(self._lib.ecl_cc_spanning_forest(
            self._h, n, nlist.numel(), _ptr(nindex), nindex.element_size(), _ptr(nlist),
            _ptr(labels), _ptr(ta), _ptr(tb), _stream_ptr(stream, d)))
        return labels, ta, tb

    def build_csr(self, n: int, src: torch.Tensor, dst: torch.Tensor, stream=None):
        """(nindex int64[n+1], nlist int32[m]) on the device: the symmetric, loop-free,
        duplicate-free CSR of the undirected edge list (src[i], dst[i]) (ecl_cc_build_csr,
        P:L223).  Synchronises the stream."""
        d = self.device
        _dev_tensor(src, "src", (torch.int32,), d)
        _dev_tensor(dst, "dst", (torch.int32,), d)
        if src.numel() != dst.numel():
            raise ValueError("src and dst must have the same length")
        E = src.numel()
        nindex = torch.empty(n + 1, dtype=torch.int64, device=d)
        cap = max(2 * E, 1)
        nlist = torch.empty(cap, dtype=torch.int32, device=d)
        m = ctypes.c_int64(0)
        self._check(self._lib.ecl_cc_build_csr(self._h, n, E, _ptr(src), _ptr(dst), _ptr(nindex),
                                               _ptr(nlist), cap, ctypes.byref(m),
                                               _stream_ptr(stream, d)))
        return nindex, nlist[:m.value].clone()

    def run_host(self, nindex, nlist, out=None, stream=None):
        """End-to-end on host buffers (numpy arrays or CPU tensors, ideally pinned)."""
        import numpy as np
        idx = torch.as_tensor(nindex)
        lst = torch.as_tensor(nlist)
        if idx.device.type != "cpu" or lst.device.type != "cpu":
            raise ValueError("run_host takes host buffers")
        if idx.dtype not in (torch.int32, torch.int64) or lst.dtype != torch.int32:
            raise TypeError("nindex must be int32/int64 and nlist int32")
        idx, lst = idx.contiguous(), lst.contiguous()
        n = idx.numel() - 1
        if out is None:
            out = torch.empty(n, dtype=torch.int32)
        out = torch.as_tensor(out)
        if out.dtype != torch.int32 or out.numel() != n or not out.is_contiguous():
            raise ValueError("out must be a contiguous int32 host buffer with n entries")
        self._check(self._lib.ecl_cc_run_host(
            self._h, n, lst.numel(), _ptr(idx), 4 if idx.dtype == torch.int32 else 8,
            _ptr(lst), _ptr(out), _stream_ptr(stream, self.device)))
        return out

    # -- multi-GPU building blocks ----------------------------------------------------
    def run_rows(self, n: int, row_lo: int, row_hi: int, nindex_rows: torch.Tensor,
                 nlist_rows: torch.Tensor, parent: Optional[torch.Tensor] = None, stream=None,
                 flatten: bool = True):
        """Local forest of rows [row_lo, row_hi) (ecl_cc_run_rows).  flatten=False leaves
        the forest unflattened (ECL_CC_OPT_STOP_AFTER = 2): enough for ecl_cc_merge on a
        peer, which saves one finalize per merge round."""
        d = self.device
        _dev_tensor(nindex_rows, "nindex_rows", (torch.int64,), d)
        _dev_tensor(nlist_rows, "nlist_rows", (torch.int32,), d)
        if nindex_rows.numel() != row_hi - row_lo + 1:
            raise ValueError("nindex_rows must hold row_hi - row_lo + 1 offsets")
        if parent is None:
            parent = torch.empty(n, dtype=torch.int32, device=d)
        _dev_tensor(parent, "parent", (torch.int32,), d)
        if not flatten:
            self.set_option("stop_after", 2)
        try:
            self._check(self._lib.ecl_cc_run_rows(self._h, n, row_lo, row_hi,
                                                  nlist_rows.numel(), _ptr(nindex_rows),
                                                  _ptr(nlist_rows), _ptr(parent),
                                                  _stream_ptr(stream, d)))
        finally:
            if not flatten:
                self.set_option("stop_after", 0)
        return parent

    def merge(self, parent: torch.Tensor, peer: torch.Tensor, v_lo: int = 0, stream=None):
        d = self.device
        _dev_tensor(parent, "parent", (torch.int32,), d)
        _dev_tensor(peer, "peer", (torch.int32,), d)
        n = parent.numel()
        self._check(self._lib.ecl_cc_merge(self._h, n, v_lo, v_lo + peer.numel(), _ptr(peer),
                                           _ptr(parent), _stream_ptr(stream, d)))
        return parent

    def finalize(self, parent: torch.Tensor, stream=None):
        d = self.device
        _dev_tensor(parent, "parent", (torch.int32,), d)
        self._check(self._lib.ecl_cc_finalize(self._h, parent.numel(), _ptr(parent),
                                              _stream_ptr(stream, d)))
        return parent

    # -- encoded forest exchange / P2P merge (ecl_cc_forest_encode, ecl_cc_merge_encoded) --
    def encode_buffers(self, n: int, cap: Optional[int] = None) -> dict:
        """Device buffers of one encoding: bits ((n+31)/32 int32 words), pairs (2*cap
        int32), meta (2 int64: pair count, D)."""
        d = self.device
        cap = n if cap is None else cap
        return {"bits": torch.empty((n + 31) // 32, dtype=torch.int32, device=d),
                "pairs": torch.empty(2 * max(cap, 1), dtype=torch.int32, device=d),
                "meta": torch.zeros(2, dtype=torch.int64, device=d), "cap": cap}

    def forest_encode(self, labels: torch.Tensor, anchor: int, enc: dict, stream=None) -> dict:
        """Encode a flattened labelling as (bitmap of label == labels[anchor], pairs)."""
        d = self.device
        _dev_tensor(labels, "labels", (torch.int32,), d)
        self._check(self._lib.ecl_cc_forest_encode(
            self._h, labels.numel(), _ptr(labels), int(anchor), _ptr(enc["bits"]),
            _ptr(enc["pairs"]), int(enc["cap"]), _ptr(enc["meta"]), _stream_ptr(stream, d)))
        return enc

    def merge_encoded(self, parent: torch.Tensor, peers, stream=None) -> torch.Tensor:
        """Hook the relations of up to 8 encodings into `parent`.  `peers` is a list of
        dicts with device pointers or tensors under bits / pairs / meta and an int cap."""
        d = self.device
        _dev_tensor(parent, "parent", (torch.int32,), d)
        k = len(peers)
        arr = lambda key: (ctypes.c_void_p * max(k, 1))(  # noqa: E731
            *[_addr(p[key]) for p in peers])
        caps = (ctypes.c_int64 * max(k, 1))(*[int(p["cap"]) for p in peers])
        self._check(self._lib.ecl_cc_merge_encoded(
            self._h, parent.numel(), k, arr("bits"), arr("pairs"), arr("meta"), caps,
            _ptr(parent), _stream_ptr(stream, d)))
        return parent

    def ipc_export(self, t: torch.Tensor) -> bytes:
        buf = ctypes.create_string_buffer(IPC_HANDLE_BYTES)
        self._check(self._lib.ecl_cc_ipc_export(_ptr(t), buf))
        return buf.raw

    def ipc_open(self, handle: bytes) -> int:
        out = ctypes.c_void_p()
        self._check(self._lib.ecl_cc_ipc_open(self.device.index, handle, ctypes.byref(out)))
        return out.value

    def ipc_close(self, ptr: int):
        self._check(self._lib.ecl_cc_ipc_close(ctypes.c_void_p(ptr)))

    # -- debug ------------------------------------------------------------------------
    def validate(self, nindex: torch.Tensor, nlist: torch.Tensor, stream=None) -> bool:
        d = self.device
        _dev_tensor(nindex, "nindex", (torch.int32, torch.int64), d)
        _dev_tensor(nlist, "nlist", (torch.int32,), d)
        st = self._lib.ecl_cc_validate(self._h, nindex.numel() - 1, nlist.numel(), _ptr(nindex),
                                       nindex.element_size(), _ptr(nlist),
                                       _stream_ptr(stream, d))
        if st == 4:
            return False
        self._check(st)
        return True

    def worklist(self):
        nf, nb = ctypes.c_int64(0), ctypes.c_int64(0)
        self._check(self._lib.ecl_cc_get_worklist(self._h, None, ctypes.byref(nf), None,
                                                  ctypes.byref(nb)))
        front = torch.empty(nf.value, dtype=torch.int32, device=self.device)
        back = torch.empty(nb.value, dtype=torch.int32, device=self.device)
        self._check(self._lib.ecl_cc_get_worklist(self._h, _ptr(front), ctypes.byref(nf),
                                                  _ptr(back), ctypes.byref(nb)))
        return front, back

    def run_info(self) -> dict:
        """Decisions of the last run (ecl_cc_get_run_info)."""
        arr = (ctypes.c_int64 * 5)()
        self._check(self._lib.ecl_cc_get_run_info(self._h, arr, 5))
        return {"lazy_init3": bool(arr[0]), "deep_forest_passes": bool(arr[1]),
                "filter": bool(arr[2]), "anchor": int(arr[3]), "fused": bool(arr[4])}

    def filter_bitmap(self):
        """(device address or None, words, anchor) of the R21 bitmap of the last run."""
        b, w, a = ctypes.c_void_p(), ctypes.c_int64(0), ctypes.c_int32(-1)
        self._check(self._lib.ecl_cc_get_filter(self._h, ctypes.byref(b), ctypes.byref(w),
                                                ctypes.byref(a)))
        return b.value, w.value, a.value

    def timing(self) -> dict:
        """Per-phase device milliseconds of the last run (needs set_option('timing', 1))."""
        arr = (ctypes.c_float * 5)()
        self._check(self._lib.ecl_cc_get_timing(self._h, arr))
        return dict(zip(PHASES, list(arr)))

    STAT_NAMES = ("cas_success", "cas_fail", "finds", "halving_stores", "edges_v_gt_u",
                  "edges_r15_same_tree", "edges_bitmap_checked", "edges_bitmap_skipped",
                  "gathers_hop1", "gathers_hop2", "bitmap_marks", "windows", "edges_queued",
                  "path_len_sum", "find_walks", "path_len_max")

    def stats(self) -> dict:
        """ECL_CC_STATS counters of the last run (ecl_cc_get_stats_ex)."""
        k = len(self.STAT_NAMES)
        arr = (ctypes.c_int64 * k)()
        self._check(self._lib.ecl_cc_get_stats_ex(self._h, arr, k))
        return dict(zip(self.STAT_NAMES, list(arr)))


_default = {}


def _handle(device) -> Handle:
    key = torch.device(device).index if device is not None else torch.cuda.current_device()
    if key not in _default:
        _default[key] = Handle(key)
    return _default[key]


def run(nindex: torch.Tensor, nlist: torch.Tensor, out: Optional[torch.Tensor] = None,
        stream=None) -> torch.Tensor:
    """Connected-component labels (min vertex ID per component) of a CSR graph on CUDA."""
    return _handle(nindex.device).run(nindex, nlist, out=out, stream=stream)


def run_host(nindex, nlist, out=None, device=None):
    """End-to-end on host arrays: H2D copy, run, D2H copy (synchronous)."""
    return _handle(device).run_host(nindex, nlist, out=out)


def _read(fn_name: str, path: str):
    import numpy as np
    lib = _load()
    n = ctypes.c_int32(0)
    e = ctypes.c_int64(0)
    a = ctypes.c_void_p()
    b = ctypes.c_void_p()
    st = getattr(lib, fn_name)(os.fsencode(path), ctypes.byref(n), ctypes.byref(e),
                               ctypes.byref(a), ctypes.byref(b))
    if st != 0:
        raise EclCCError(st, lib.ecl_cc_io_last_error().decode())
    try:
        k = e.value
        src = np.ctypeslib.as_array((ctypes.c_int32 * max(k, 1)).from_address(a.value))[:k].copy()
        dst = np.ctypeslib.as_array((ctypes.c_int32 * max(k, 1)).from_address(b.value))[:k].copy()
    finally:
        lib.ecl_cc_free_host(a)
        lib.ecl_cc_free_host(b)
    return n.value, src, dst


def read_mtx(path: str):
    """(n, src, dst) numpy int32 edge list of a MatrixMarket coordinate file (ecl_cc_read_mtx;
    host-only C reader, no GPU needed)."""
    return _read("ecl_cc_read_mtx", path)


def read_edgelist(path: str):
    """(n, src, dst) of a SNAP-style whitespace edge list (ecl_cc_read_edgelist)."""
    return _read("ecl_cc_read_edgelist", path)

"""CPU oracle for ECL-CC connected components (ctypes wrapper over oracle/oracle.c).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this module.  The product package
``paper_conf_hpdc_jaiganeshb18_b200`` never imports it, and it never imports the product.

Functions (each follows the passage cited in oracle/oracle.c):
  bfs(nindex, nlist)      -> (labels, ncc)   O1, P:L51 (§1) serial BFS, ascending sources
  uf(nindex, nlist)       -> (labels, ncc)   O2, P:L53 (§1) serial union-find, union by min
  init3(nindex, nlist)    -> parent          Init3, P:L141 (§3)
  check(nindex, nlist, labels, ncc) -> int   invariants I1–I3; 0 = ok
  check_forest(nindex, nlist, labels, ta, tb) -> int   spanning-forest definition; 0 = ok
  bfs_forest(nindex, nlist) -> (ta, tb, ncc)  the BFS tree edges of O1 (a valid forest)
  build_csr(n, src, dst) -> (nindex, nlist)  P:L223 input preparation (loops, multi-edges,
                                              back edges), rows ascending

Inputs are numpy arrays (CSR: ``nindex`` of n+1 offsets, int32 or int64; ``nlist`` int32).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")


def _cpu_tag() -> str:
    """-march=native code is host specific: key the library by the host CPU model."""
    import hashlib
    import platform
    model = platform.machine()
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith(("model name", "flags")):
                    model += line
    except OSError:
        pass
    return hashlib.sha1(model.encode()).hexdigest()[:10]


_LIB = os.path.join(_HERE, f"liboracle-{_cpu_tag()}.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with the paper's CPU flags (-O3 -march=native)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=native", "-std=c11", "-shared", "-fPIC",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        p = ctypes.c_void_p
        lib.oracle_bfs.argtypes = [ctypes.c_int32, p, p, p]
        lib.oracle_bfs.restype = ctypes.c_int64
        lib.oracle_uf.argtypes = [ctypes.c_int32, p, p, p]
        lib.oracle_uf.restype = ctypes.c_int64
        lib.oracle_init3.argtypes = [ctypes.c_int32, p, p, p]
        lib.oracle_init3.restype = None
        lib.oracle_check.argtypes = [ctypes.c_int32, p, p, p, ctypes.c_int64]
        lib.oracle_check.restype = ctypes.c_int
        lib.oracle_check_forest.argtypes = [ctypes.c_int32, p, p, p, p, p]
        lib.oracle_check_forest.restype = ctypes.c_int
        lib.oracle_bfs_forest.argtypes = [ctypes.c_int32, p, p, p, p]
        lib.oracle_bfs_forest.restype = ctypes.c_int64
        lib.oracle_build_csr.argtypes = [ctypes.c_int32, ctypes.c_int64, p, p, p, p]
        lib.oracle_build_csr.restype = ctypes.c_int64
        _lib = lib
    return _lib


def _csr(nindex, nlist):
    nindex = np.ascontiguousarray(np.asarray(nindex), dtype=np.int64)
    nlist = np.ascontiguousarray(np.asarray(nlist), dtype=np.int32)
    n = nindex.shape[0] - 1
    if n < 0:
        raise ValueError("nindex must hold n+1 offsets")
    if nindex[0] != 0 or nindex[-1] != nlist.shape[0]:
        raise ValueError("nindex[0] must be 0 and nindex[n] must equal len(nlist)")
    return n, nindex, nlist


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def bfs(nindex, nlist):
    n, nindex, nlist = _csr(nindex, nlist)
    out = np.empty(n, dtype=np.int32)
    ncc = _load().oracle_bfs(n, _ptr(nindex), _ptr(nlist), _ptr(out))
    if ncc < 0:
        raise MemoryError("oracle_bfs failed")
    return out, int(ncc)


def uf(nindex, nlist):
    n, nindex, nlist = _csr(nindex, nlist)
    out = np.empty(n, dtype=np.int32)
    ncc = _load().oracle_uf(n, _ptr(nindex), _ptr(nlist), _ptr(out))
    return out, int(ncc)


def init3(nindex, nlist):
    n, nindex, nlist = _csr(nindex, nlist)
    out = np.empty(n, dtype=np.int32)
    _load().oracle_init3(n, _ptr(nindex), _ptr(nlist), _ptr(out))
    return out


def check(nindex, nlist, labels, ncc_expected: int) -> int:
    n, nindex, nlist = _csr(nindex, nlist)
    labels = np.ascontiguousarray(np.asarray(labels), dtype=np.int32)
    if labels.shape[0] != n:
        raise ValueError("labels must have n entries")
    return int(_load().oracle_check(n, _ptr(nindex), _ptr(nlist), _ptr(labels), int(ncc_expected)))


def check_forest(nindex, nlist, labels, ta, tb) -> int:
    """0 if the per-vertex edge slots (ta, tb) form a spanning forest of the graph (labels =
    the oracle's min-ID labels, which fix the (-1, -1) slots of component minima)."""
    n, nindex, nlist = _csr(nindex, nlist)
    arrs = [np.ascontiguousarray(np.asarray(a), dtype=np.int32) for a in (labels, ta, tb)]
    if any(a.shape[0] != n for a in arrs):
        raise ValueError("labels, ta and tb must have n entries")
    return int(_load().oracle_check_forest(n, _ptr(nindex), _ptr(nlist), *(_ptr(a) for a in arrs)))


def bfs_forest(nindex, nlist):
    n, nindex, nlist = _csr(nindex, nlist)
    ta = np.empty(n, dtype=np.int32)
    tb = np.empty(n, dtype=np.int32)
    ncc = _load().oracle_bfs_forest(n, _ptr(nindex), _ptr(nlist), _ptr(ta), _ptr(tb))
    if ncc < 0:
        raise MemoryError("oracle_bfs_forest failed")
    return ta, tb, int(ncc)


def build_csr(n: int, src, dst):
    src = np.ascontiguousarray(np.asarray(src), dtype=np.int32)
    dst = np.ascontiguousarray(np.asarray(dst), dtype=np.int32)
    if src.shape != dst.shape:
        raise ValueError("src and dst must have the same length")
    E = src.shape[0]
    nindex = np.empty(n + 1, dtype=np.int64)
    nlist = np.empty(max(2 * E, 1), dtype=np.int32)
    m = _load().oracle_build_csr(n, E, _ptr(src), _ptr(dst), _ptr(nindex), _ptr(nlist))
    if m < 0:
        raise ValueError("oracle_build_csr: vertex ID out of range or allocation failure")
    return nindex, nlist[:m].copy()

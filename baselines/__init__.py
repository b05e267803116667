"""The paper's CPU versions of ECL-CC (ECL-CCOMP; ECL-CCSER) as CPU
comparison points for bench.py.  Not the oracle and not the product:
plain C + OpenMP in baselines/ecl_cc_cpu.c, compiled with the paper's flags."""
from __future__ import annotations

import ctypes
import hashlib
import os
import platform
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ecl_cc_cpu.c")


def _tag() -> str:
    model = platform.machine()
    try:
        with open("/proc/cpuinfo") as f:
            model += "".join(ln for ln in f if ln.startswith(("model name", "flags")))
    except OSError:
        pass
    return hashlib.sha1(model.encode()).hexdigest()[:10]


_LIB = os.path.join(_HERE, f"libecl_cc_cpu-{_tag()}.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=native", "-fopenmp", "-std=c11", "-shared",
                               "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        p = ctypes.c_void_p
        lib.eclcc_omp.argtypes = [ctypes.c_int32, p, p, p, ctypes.c_int]
        lib.eclcc_omp.restype = None
        lib.eclcc_ser.argtypes = [ctypes.c_int32, p, p, p]
        lib.eclcc_ser.restype = None
        _lib = lib
    return _lib


def _csr(nindex, nlist):
    nindex = np.ascontiguousarray(np.asarray(nindex), dtype=np.int64)
    nlist = np.ascontiguousarray(np.asarray(nlist), dtype=np.int32)
    return nindex.shape[0] - 1, nindex, nlist


def omp(nindex, nlist, threads: int = 0) -> np.ndarray:
    """ECL-CCOMP labels (threads = 0: all host cores)."""
    n, nindex, nlist = _csr(nindex, nlist)
    out = np.empty(n, dtype=np.int32)
    t = threads or os.cpu_count() or 1
    p = lambda a: a.ctypes.data_as(ctypes.c_void_p)  # noqa: E731
    _load().eclcc_omp(n, p(nindex), p(nlist), p(out), t)
    return out


def ser(nindex, nlist) -> np.ndarray:
    """ECL-CCSER labels."""
    n, nindex, nlist = _csr(nindex, nlist)
    out = np.empty(n, dtype=np.int32)
    p = lambda a: a.ctypes.data_as(ctypes.c_void_p)  # noqa: E731
    _load().eclcc_ser(n, p(nindex), p(nlist), p(out))
    return out

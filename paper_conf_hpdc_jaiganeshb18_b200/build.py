"""Build libecl_cc.so (and the ECL_CC_STATS debug variant) for sm_100a with nvcc.

Run ``python -m paper_conf_hpdc_jaiganeshb18_b200.build`` or call ``build()``.  The
libraries are written next to this file (in-tree) so they travel with the repo snapshot.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
SOURCES = [os.path.join(CSRC, "ecl_cc.cu"), os.path.join(CSRC, "ecl_cc_csr.cu"),
           os.path.join(CSRC, "ecl_cc_io.cpp")]
DEPS = SOURCES + [os.path.join(CSRC, "ecl_cc_kernels.cuh"), os.path.join(CSRC, "ecl_cc_ctx.h"),
                  os.path.join(INCLUDE, "ecl_cc.h")]

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
         "-Xcompiler", "-fvisibility=hidden", "--expt-relaxed-constexpr",
         "-I" + INCLUDE, "-I" + CSRC]

VARIANTS = {
    "libecl_cc.so": [],
    "libecl_cc_stats.so": ["-DECL_CC_STATS"],
}


def lib_path(name: str = "libecl_cc.so") -> str:
    return os.path.join(PKG, name)


def _stale(out: str) -> bool:
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(d) > t for d in DEPS)


def build(force: bool = False, verbose: bool = False) -> list:
    built = []
    for name, extra in VARIANTS.items():
        out = lib_path(name)
        if not force and not _stale(out):
            continue
        tmp = out + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, *FLAGS, *extra, *SOURCES, "-o", tmp]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
            print(" ".join(cmd), file=sys.stderr)
        subprocess.check_call(cmd)
        os.replace(tmp, out)
        built.append(out)
    return built


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)

"""Measure the L2 random-sector ceiling (tools/l2_ceiling.cu) on this GPU.

    python tools/l2_ceiling.py      -> one JSON line (loads per second per pattern)
"""
import ctypes
import json
import os
import subprocess
import sys

import torch

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SO = os.path.join(ROOT, "build", "l2_ceiling.so")


def build():
    os.makedirs(os.path.dirname(SO), exist_ok=True)
    src = os.path.join(HERE, "l2_ceiling.cu")
    if not os.path.exists(SO) or os.path.getmtime(SO) < os.path.getmtime(src):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode",
                               "arch=compute_100a,code=sm_100a", "-O3", "-shared",
                               "-Xcompiler", "-fPIC", src, "-o", SO])


def timed(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    build()
    lib = ctypes.CDLL(SO)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    out = torch.zeros(1, dtype=torch.int32, device="cuda")
    res = {"sms": sms}
    for mb in (16, 64, 512):
        words = mb * 2 ** 20 // 4
        table = torch.randint(0, 2 ** 31, (words,), dtype=torch.int32, device="cuda")
        P = 2 ** 30
        for gm in (8, 16):
            ms = timed(lambda: lib.l2c_random(ctypes.c_longlong(P), ctypes.c_void_p(table.data_ptr()),
                                              ctypes.c_ulonglong(words), ctypes.c_void_p(out.data_ptr()),
                                              sms * gm))
            res[f"random_{mb}MB_grid{gm}_Gloads_s"] = round(P / ms / 1e6, 1)
        del table
    # the R21 probe pattern at C5 scale: bitmap of 2^27 bits, 2^30 streamed entries
    n = 2 ** 27
    table = torch.zeros(n // 32, dtype=torch.int32, device="cuda")
    E = 2 ** 30
    lst = torch.randint(0, n, (E,), dtype=torch.int32, device="cuda")
    ms = timed(lambda: lib.l2c_probe(ctypes.c_longlong(E), ctypes.c_void_p(lst.data_ptr()),
                                     ctypes.c_void_p(table.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                     sms * 8))
    res["probe_pattern_ms_per_2^30_entries"] = round(ms, 3)
    res["probe_pattern_entries_G_s"] = round(E / ms / 1e6, 1)
    res["probe_pattern_sectors_G_s"] = round((E / 2 + E * 4 / 32) / ms / 1e6, 1)
    if "--sweep" in sys.argv:
        for U in (4, 8, 16):
            for fl, nm in ((0, "ca"), (1, "cg"), (2, "noalloc"), (3, "relaxed_gpu")):
                for gm in (4, 8):
                    ms = timed(lambda: lib.l2c_probe_v(ctypes.c_longlong(E), ctypes.c_void_p(lst.data_ptr()),
                                                       ctypes.c_void_p(table.data_ptr()),
                                                       ctypes.c_void_p(out.data_ptr()), sms * gm, fl, U))
                    res[f"probe_U{U}_{nm}_grid{gm}_entries_G_s"] = round(E / ms / 1e6, 1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()

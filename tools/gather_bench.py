"""Random-gather ceiling vs the hook kernels on one config (see gather_bench.cu)."""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_hpdc_jaiganeshb18_b200 as ecl  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
g = gg.make_config(cfg, device="cuda")
lib = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "build",
                               "gather_bench.so"))
src = torch.repeat_interleave(torch.arange(g.n, device="cuda", dtype=torch.int32), g.degrees())
h = ecl.Handle(0)
labels = h.run(g.nindex, g.nlist)
out = torch.zeros(1, dtype=torch.int64, device="cuda")
hooked = int((g.nlist < src).sum())
res = {"config": cfg, "m": g.m, "hooked": hooked}
for hint in (0, 1):
    for _ in range(2):
        lib.gather_run(hint, ctypes.c_longlong(g.m), ctypes.c_void_p(src.data_ptr()),
                       ctypes.c_void_p(g.nlist.data_ptr()), ctypes.c_void_p(labels.data_ptr()),
                       ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(0))
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(3):
        lib.gather_run(hint, ctypes.c_longlong(g.m), ctypes.c_void_p(src.data_ptr()),
                       ctypes.c_void_p(g.nlist.data_ptr()), ctypes.c_void_p(labels.data_ptr()),
                       ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(0))
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    res[f"gather_ms_hint{hint}"] = round(ms, 3)
    res[f"gathers_per_s_hint{hint}"] = round(hooked / ms / 1e6, 1)  # G/s
print(json.dumps(res))

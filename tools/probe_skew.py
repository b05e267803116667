"""How concentrated are the hook kernels' R21 bitmap probes?  For every entry (v,u) with
v > u in rows of degree > t1 (hook_warp/hook_block), count probes per bitmap word u >> 5
and report the share of probes that the K most-probed words receive.
    python tools/probe_skew.py C5 [scale_down]"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
sd = int(sys.argv[2]) if len(sys.argv) > 2 else 0
g = gg.make_config(cfg, seed=1, device="cuda", scale_down=sd)
n = g.n
ni = g.nindex.to(torch.int64)
deg = ni[1:] - ni[:-1]
words = torch.zeros((n + 31) // 32, dtype=torch.int64, device="cuda")
chunk = 1 << 28
for a in range(0, g.m, chunk):
    pos = torch.arange(a, min(g.m, a + chunk), device="cuda", dtype=torch.int64)
    v = torch.searchsorted(ni, pos, right=True) - 1
    u = g.nlist[a:a + chunk].to(torch.int64)
    keep = (v > u) & (deg[v] > 16)
    words.index_add_(0, u[keep] >> 5, torch.ones_like(u[keep]))
    del pos, v, u, keep
tot = int(words.sum())
s, _ = torch.sort(words, descending=True)
c = torch.cumsum(s, 0)
out = {"config": cfg, "n": n, "probes": tot, "words": int(words.numel())}
for K in [1024, 4096, 16384, 65536, 262144, 1 << 20]:
    out[f"top{K}"] = round(float(c[min(K, len(c)) - 1]) / tot, 4)
print(json.dumps(out))

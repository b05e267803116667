"""How many thread-bin active vertices need no hook work at all (every entry u < v is the
Init3 parent, so R15 skips it)?  Split by whether init already reads the whole row
(deg <= 4).   python tools/thread_work.py C5 [scale_down]"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
sd = int(sys.argv[2]) if len(sys.argv) > 2 else 0
g = gg.make_config(cfg, seed=1, device="cuda", scale_down=sd)
n, m = g.n, g.m
ni = g.nindex.to(torch.int64)
deg = ni[1:] - ni[:-1]
# rows are sorted ascending: Init3 parent = first entry if it is smaller
first = g.nlist[ni[:-1].clamp(max=m - 1)].to(torch.int64)
v = torch.arange(n, device="cuda")
active = (deg > 0) & (first < v)
lt = torch.zeros(n, dtype=torch.int64, device="cuda")
chunk = 1 << 28
for a in range(0, m, chunk):
    pos = torch.arange(a, min(m, a + chunk), device="cuda", dtype=torch.int64)
    rows = torch.searchsorted(ni, pos, right=True) - 1
    u = g.nlist[a:a + chunk].to(torch.int64)
    other = (u < rows) & (u != first[rows])          # smaller and not the Init3 parent
    lt.index_add_(0, rows[other], torch.ones(int(other.sum()), dtype=torch.int64, device="cuda"))
    del pos, rows, u, other
thr = active & (deg <= 16)
nowork = thr & (lt == 0)
out = {"config": cfg, "n": n, "thread_active": int(thr.sum()),
       "no_work": int(nowork.sum()), "no_work_deg_le4": int((nowork & (deg <= 4)).sum()),
       "thread_active_deg_le4": int((thr & (deg <= 4)).sum()),
       "entries_of_no_work_rows": int(deg[nowork].sum()),
       "thread_entries": int(deg[thr].sum())}
print(json.dumps(out))

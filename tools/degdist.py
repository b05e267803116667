"""Degree distribution of a config: rows / entries above degree thresholds, and how many
entries of rows <= T point at rows > T (hub-leaf edges).  python tools/degdist.py C5"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
sd = int(sys.argv[2]) if len(sys.argv) > 2 else 0
g = gg.make_config(cfg, seed=1, device="cuda", scale_down=sd)
ni = g.nindex.to(torch.int64)
deg = ni[1:] - ni[:-1]
n, m = g.n, g.m
out = {"config": cfg, "n": n, "m": m}
rows = []
for T in [16, 64, 352, 1024, 4096, 16384, 65536]:
    hub = deg > T
    nh = int(hub.sum())
    ent = int(deg[hub].sum())
    # entries of non-hub rows whose neighbour is a hub, split by direction
    src = torch.repeat_interleave(torch.arange(n, device="cuda"), deg)
    nl = g.nlist.to(torch.int64)
    leaf_side = ~hub[src]
    to_hub = hub[nl] & leaf_side
    up = int((to_hub & (nl > src)).sum())
    hh = int((hub[src] & hub[nl]).sum())
    rows.append({"T": T, "hubs": nh, "hub_entries": ent, "leaf_to_hub_entries": int(to_hub.sum()),
                 "leaf_to_larger_hub": up, "hub_hub_entries": hh})
    del src, nl, leaf_side, to_hub
    torch.cuda.empty_cache()
out["rows"] = rows
print(json.dumps(out))

"""Single-GPU emulation of the 2/4/8-GPU path — a PROJECTION, not a
measurement: this run has one B200.

For G ranks: the row partition of bench.py (partition_rows), every rank's local forest
(ecl_cc_run_rows) timed with CUDA events one rank after another on this GPU, then the
binomial-tree merge rounds (ecl_cc_merge on the receiving rank's forest, timed; only rank
0 flattens at the end, as dist.forest_merge does), and the NCCL transfer of n int32
entries per round modelled at --link-gbs (NVLink 5: 900 GB/s per direction nominal).  The
merge overlaps chunk c+1's transfer with chunk c's hook, so a round is modelled as
transfer + merge/chunks.  Projected step = max over ranks of the local forest + the sum
of rounds + rank 0's finalize.  The merged labels are checked against the single-GPU
labels.  --even uses the plain m/G entry split instead of the work-weighted one.

    python tools/mgpu_emulate.py [--config C5] [--gpus 1,2,4,8] [--link-gbs 750] [--order 2]
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg  # noqa: E402
import paper_conf_hpdc_jaiganeshb18_b200 as ecl  # noqa: E402
from paper_conf_hpdc_jaiganeshb18_b200 import dist as edist  # noqa: E402


def timed(fn, reps=3):
    best = None
    for _ in range(reps):
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record()
        out = fn()
        b.record()
        torch.cuda.synchronize()
        t = a.elapsed_time(b)
        best = t if best is None else min(best, t)
    return best, out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--gpus", default="1,2,4,8")
    ap.add_argument("--link-gbs", type=float, default=750.0)
    ap.add_argument("--chunks", type=int, default=4)
    ap.add_argument("--even", action="store_true")
    ap.add_argument("--order", type=int, default=2, help="ECL_CC_OPT_ORDER of every run")
    args = ap.parse_args()
    g = gg.make_config(args.config, seed=1, device="cuda")
    n, m = g.n, g.m
    h = ecl.Handle(0)
    h.set_option("order", args.order)
    nidx64 = g.nindex.to(torch.int64)
    ref = torch.empty(n, dtype=torch.int32, device="cuda")
    t1, _ = timed(lambda: h.run(g.nindex, g.nlist, out=ref))
    res = {"config": args.config, "n": n, "m": m, "single_gpu_ms": round(t1, 4),
           "link_gbs_model": args.link_gbs, "chunks": args.chunks, "kind": "projection",
           "rows": []}
    wts = None if args.even else edist.row_weights(nidx64, g.nlist)
    res["partition"] = "entries" if args.even else "row_weights"
    for G in [int(x) for x in args.gpus.split(",")]:
        bounds = edist.partition_rows(nidx64.cpu(), G, weights=wts)
        forests, t_rank = [], []
        for r in range(G):
            lo, hi = bounds[r], bounds[r + 1]
            idx, lst = edist.slice_rows(nidx64, g.nlist, lo, hi)
            par = torch.empty(n, dtype=torch.int32, device="cuda")
            t, _ = timed(lambda: h.run_rows(n, lo, hi, idx, lst, parent=par, flatten=(G == 1)))
            t_rank.append(t)
            forests.append(par)
            del idx, lst
        rounds = {}
        for (rd, send, recv) in edist.tree_schedule(G):
            base = forests[recv].clone()

            def mrg():
                forests[recv].copy_(base)
                h.merge(forests[recv], forests[send])
                return None
            copy_t, _ = timed(lambda: forests[recv].copy_(base))
            t_m, _ = timed(mrg)
            t_m = max(t_m - copy_t, 0.0)
            forests[recv].copy_(base)
            h.merge(forests[recv], forests[send])
            xfer = n * 4 / (args.link_gbs * 1e9) * 1e3
            rt = xfer + t_m / args.chunks
            rounds.setdefault(rd, []).append({"send": send, "recv": recv, "merge_ms": round(t_m, 4),
                                              "transfer_ms_model": round(xfer, 4),
                                              "round_ms": round(rt, 4)})
            del base
        t_fin = 0.0
        if G > 1:
            t_fin, _ = timed(lambda: h.finalize(forests[0]), reps=1)
        torch.cuda.synchronize()
        ok = bool(torch.equal(forests[0], ref))
        t_rounds = sum(max(x["round_ms"] for x in v) for v in rounds.values())
        proj = max(t_rank) + t_rounds + t_fin
        res["rows"].append({"gpus": G, "rank_forest_ms": [round(x, 4) for x in t_rank],
                            "merge_rounds": rounds, "final_flatten_ms": round(t_fin, 4),
                            "projected_ms": round(proj, 4),
                            "projected_Medges_s": round(m / proj / 1e3, 1),
                            "projected_speedup": round(t1 / proj, 3), "labels_exact": ok})
        del forests
        torch.cuda.empty_cache()
    print(json.dumps(res))


if __name__ == "__main__":
    main()

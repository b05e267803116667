"""Run-to-run spread of one config: N back-to-back runs timed with CUDA events (no
flush), optionally with the stats build to correlate time with CAS/find counters.

    python tools/variance.py --config C3 --runs 30 [--stats] [--opt name=value ...]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_hpdc_jaiganeshb18_b200 as ecl  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--runs", type=int, default=30)
    ap.add_argument("--stats", action="store_true")
    ap.add_argument("--opt", nargs="*", default=[])
    args = ap.parse_args()
    g = gg.make_config(args.config, seed=1, device="cuda")
    h = ecl.Handle(0, stats=args.stats)
    for o in args.opt:
        k, v = o.split("=")
        h.set_option(k, int(v))
    out = torch.empty(g.n, dtype=torch.int32, device="cuda")
    h.run(g.nindex, g.nlist, out=out)
    rows = []
    for _ in range(args.runs):
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record()
        h.run(g.nindex, g.nlist, out=out)
        b.record()
        b.synchronize()
        r = {"ms": round(a.elapsed_time(b), 4)}
        if args.stats:
            st = h.stats()
            r.update({k: st[k] for k in ("cas_success", "cas_fail", "finds", "halving_stores",
                                          "edges_queued", "path_len_max")})
        rows.append(r)
    ms = [r["ms"] for r in rows]
    print(json.dumps({"config": args.config, "opts": args.opt, "stats": args.stats,
                      "min": min(ms), "median": statistics.median(ms), "max": max(ms),
                      "runs": rows if args.stats else ms}))


if __name__ == "__main__":
    main()

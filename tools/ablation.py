"""Paper ablations on B200: Figs. 7, 8, 9 and Table 4 of the paper
(P:L235-L343).

For each config: the relative runtime of Init1/Init2 vs Init3 (Fig. 7), Jump1/2/3 vs
Jump4 (Fig. 8), Fini1/2 vs Fini3 (Fig. 9) — whole runs timed with CUDA events (median of
--reps, L2 flushed between runs when the graph fits in L2), values > 1 = slower than
ECL-CC's choice (the paper's convention) — and, from the -DECL_CC_STATS build, the
average and maximum find_repres path length of every variant (Table 4).
Every variant's labels must equal the default's.

    python tools/ablation.py [--reps 7] [C1 C2 C3 C4 C5]
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

# Jump1-3 exist only on the plain path (one find + hook per edge, no R19/R22 batching),
# so "Jump4_plain" (batch 0) is their like-for-like baseline: relative_to_jump4_plain
VARIANTS = [("base", {}), ("Init1", {"init": 1}), ("Init2", {"init": 2}),
            ("Jump4_plain", {"batch": 0}),
            ("Jump1", {"jump": 1}), ("Jump2", {"jump": 2}), ("Jump3", {"jump": 3}),
            ("Fini1", {"fini": 1}), ("Fini2", {"fini": 2}),
            ("separate_Init3_pass", {"fuse_init": 0})]
DEF = {"init": 3, "jump": 4, "fini": 3, "batch": 1, "fuse_init": 2}
L2 = 126 << 20


def run(h, g, opts, reps, flush):
    for k, v in DEF.items():
        h.set_option(k, opts.get(k, v))
    out = torch.empty(g.n, dtype=torch.int32, device="cuda")
    h.run(g.nindex, g.nlist, out=out)
    ts = []
    for _ in range(reps):
        if flush is not None:
            flush.add_(1)
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record()
        h.run(g.nindex, g.nlist, out=out)
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts), out


def paths(hs, g, opts):
    for k, v in DEF.items():
        hs.set_option(k, opts.get(k, v))
    hs.run(g.nindex, g.nlist)
    st = hs.stats()
    w = st["find_walks"]
    return {"avg_path": round(st["path_len_sum"] / w, 3) if w else None,
            "max_path": st["path_len_max"], "find_walks": w,
            "halving_stores": st["halving_stores"], "cas_success": st["cas_success"],
            "cas_fail": st["cas_fail"]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=7)
    ap.add_argument("--skip", default="", help="variants to skip, e.g. Jump3")
    ap.add_argument("configs", nargs="*")
    args = ap.parse_args()
    cfgs = args.configs or ["C1", "C2", "C3", "C4", "C5"]
    skip = set(args.skip.split(",")) if args.skip else set()
    h = ecl.Handle(0)
    hs = ecl.Handle(0, stats=True)
    for c in cfgs:
        g = gg.make_config(c, device="cuda")
        flush = torch.zeros(64 << 20, dtype=torch.int32, device="cuda") if g.m * 4 < 2 * L2 \
            else None
        base, ref = run(h, g, {}, args.reps, flush)
        row = {"config": c, "n": g.n, "m": g.m, "base_ms": round(base, 4),
               "relative_runtime": {}, "paths": {"base": paths(hs, g, {})}}
        for name, opts in VARIANTS[1:]:
            if name in skip:
                continue
            t, out = run(h, g, opts, max(3, args.reps // 2) if name == "Jump3" else args.reps,
                         flush)
            assert torch.equal(out, ref), (c, name)
            row["relative_runtime"][name] = round(t / base, 3)
            row.setdefault("ms", {})[name] = round(t, 4)
            row["paths"][name] = paths(hs, g, opts)
        jp = row.get("ms", {}).get("Jump4_plain")
        if jp:
            row["relative_to_jump4_plain"] = {k: round(row["ms"][k] / jp, 3)
                                              for k in ("Jump1", "Jump2", "Jump3")
                                              if k in row["ms"]}
        print(json.dumps(row), flush=True)
        del g, flush
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()

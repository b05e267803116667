"""Paper ablations on B200: Figs. 7, 8, 9 of the paper.

Relative runtime of Init1/Init2 vs Init3, Jump1/2/3 vs Jump4, Fini1/2 vs Fini3, per config;
values > 1 mean slower than ECL-CC's choice (the paper's convention).
    python tools/ablation.py [C1 C2 C3 C4 C5]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_hpdc_jaiganeshb18_b200 as ecl  # noqa: E402

VARIANTS = [("base", {}), ("Init1", {"init": 1}), ("Init2", {"init": 2}),
            ("Jump1", {"jump": 1}), ("Jump2", {"jump": 2}), ("Jump3", {"jump": 3}),
            ("Fini1", {"fini": 1}), ("Fini2", {"fini": 2})]
DEF = {"init": 3, "jump": 4, "fini": 3}


def run(h, g, opts, reps=5):
    for k, v in DEF.items():
        h.set_option(k, opts.get(k, v))
    out = torch.empty(g.n, dtype=torch.int32, device="cuda")
    h.run(g.nindex, g.nlist, out=out)
    best = None
    for _ in range(reps):
        h.run(g.nindex, g.nlist, out=out)
        t = sum(h.timing().values())
        best = t if best is None else min(best, t)
    return best, out


def main():
    cfgs = sys.argv[1:] or ["C1", "C2", "C3", "C4"]
    h = ecl.Handle(0)
    h.set_option("timing", 1)
    for c in cfgs:
        g = gg.make_config(c, device="cuda")
        base, ref = run(h, g, {})
        row = {"config": c, "base_ms": round(base, 4)}
        for name, opts in VARIANTS[1:]:
            t, out = run(h, g, opts, reps=3 if name == "Jump3" else 5)
            assert torch.equal(out, ref), (c, name)
            row[name] = round(t / base, 3)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()

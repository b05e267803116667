"""Small cases for compute-sanitizer: memcheck / racecheck / synccheck.

    compute-sanitizer --tool racecheck python tools/sanitize_cases.py [--quick]

Runs the hand-built graphs (clean and raw: loops, duplicates, unsorted rows) and C1 / a
scaled C2 / C4 / C5 through ecl_cc_run, ecl_cc_run_i64, the spanning forest and the
multi-GPU building blocks (run_rows -> merge -> finalize), under kernel orders 0 and 2,
with the R23 prejump passes forced on (cooperative grid barrier) and off, and the R21
bitmap filter forced on; every result is compared with oracle O1.  Exit code 1 on any
mismatch.
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402
import paper_conf_hpdc_jaiganeshb18_b200 as ecl  # noqa: E402
from paper_conf_hpdc_jaiganeshb18_b200 import dist as edist  # noqa: E402


def cases(quick):
    from test_gpu_parity import hand_graphs
    from test_gpu_raw_csr import hand_raw_graphs
    G = [g for g in hand_graphs() if g.n <= 5000] + hand_raw_graphs()[:5]
    G.append(gg.make_config("C1", seed=1))
    G.append(gg.inject_loops_dups(gg.make_config("C1", seed=2, scale_down=2), seed=1))
    if not quick:
        G.append(gg.make_config("C2", seed=1, scale_down=10))
        G.append(gg.make_config("C4", seed=1, scale_down=12))
        G.append(gg.make_config("C5", seed=1, scale_down=14))
    return G


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--variants", action="store_true",
                    help="also the ablation paths (Jump1-3, batch 0, Init1/2, Fini1/2) and "
                         "the R31 quad engine")
    args = ap.parse_args()
    bad = 0
    runs = 0
    with ecl.Handle(0) as h:
        for g in cases(args.quick):
            gd = g.to("cuda")
            expect, _ = oracle.bfs(*g.numpy())
            for order in (0, 2):
                for prejump in (0, 1):
                    for filt in (0, 1):
                        h.set_option("order", order).set_option("prejump", prejump)
                        h.set_option("filter", filt)
                        for idx in (gd.nindex, gd.nindex.to(torch.int64)):
                            out = h.run(idx, gd.nlist)
                            torch.cuda.synchronize()
                            runs += 1
                            if not np.array_equal(out.cpu().numpy(), expect):
                                print(f"MISMATCH {g.name} order={order} prejump={prejump} "
                                      f"filter={filt} idx={idx.dtype}", flush=True)
                                bad += 1
            if args.variants:
                for opts in (dict(jump=1), dict(jump=2), dict(jump=3), dict(batch=0),
                             dict(init=1, fini=1), dict(init=2, fini=2), dict(vec=1),
                             dict(vec=1, thresh_thread=2, thresh_warp=20, filter=1)):
                    for k, v in opts.items():
                        h.set_option(k, v)
                    out = h.run(gd.nindex, gd.nlist)
                    torch.cuda.synchronize()
                    runs += 1
                    if not np.array_equal(out.cpu().numpy(), expect):
                        print(f"MISMATCH {g.name} {opts}", flush=True)
                        bad += 1
                    for k in opts:
                        h.set_option(k, {"jump": 4, "batch": 1, "init": 3, "fini": 3, "vec": 2,
                                         "thresh_thread": 16, "thresh_warp": 352,
                                         "filter": filt}[k])
            h.set_option("order", 2).set_option("prejump", 1).set_option("filter", 2)
            lab, ta, tb = h.spanning_forest(gd.nindex, gd.nlist)
            torch.cuda.synchronize()
            runs += 1
            if not np.array_equal(lab.cpu().numpy(), expect) or oracle.check_forest(
                    *g.numpy(), expect, ta.cpu().numpy(), tb.cpu().numpy()) != 0:
                print(f"FOREST MISMATCH {g.name}", flush=True)
                bad += 1
            # multi-GPU building blocks: 3 fake ranks, tree merge, one flatten
            nidx64 = gd.nindex.to(torch.int64)
            b = edist.partition_rows(nidx64.cpu(), 3)
            forests = []
            for r in range(3):
                i, l_ = edist.slice_rows(nidx64, gd.nlist, b[r], b[r + 1])
                forests.append(h.run_rows(g.n, b[r], b[r + 1], i, l_, flatten=False))
            f0 = forests[0].clone()
            for (_, s, rcv) in edist.tree_schedule(3):
                h.merge(forests[rcv], forests[s])
            h.finalize(forests[0])
            torch.cuda.synchronize()
            runs += 1
            if not np.array_equal(forests[0].cpu().numpy(), expect):
                print(f"MERGE MISMATCH {g.name}", flush=True)
                bad += 1
            # encoded merge of ranks 1, 2 into rank 0
            encs = []
            for r in (1, 2):
                i, l_ = edist.slice_rows(nidx64, gd.nlist, b[r], b[r + 1])
                f = h.run_rows(g.n, b[r], b[r + 1], i, l_)
                e = h.encode_buffers(g.n)
                h.forest_encode(f, edist.row_anchor(i, b[r]), e)
                encs.append(e)
            h.merge_encoded(f0, encs)
            h.finalize(f0)
            torch.cuda.synchronize()
            runs += 1
            if not np.array_equal(f0.cpu().numpy(), expect):
                print(f"ENCODED MERGE MISMATCH {g.name}", flush=True)
                bad += 1
    print(f"sanitize_cases: {runs} runs, {bad} mismatches", flush=True)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()

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
                                 [--merge tree,encoded]

--merge encoded projects dist.EncodedMerge: every rank g > 0 flattens
its local forest and encodes it (ecl_cc_forest_encode: bitmap of its anchor's class +
pairs), rank 0 merges all encodings in one ecl_cc_merge_encoded call (kernels timed here
on local copies) and flattens once.  In the p2p mode the merge kernels read the peers'
buffers over NVLink, so the merge is modelled as max(kernel time, encoded bytes / link
bandwidth into rank 0); the compact mode adds the transfer instead.
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


def depth_stats(parent):
    """Mean / max depth (pointers to the root) of a forest, by pointer doubling."""
    anc = parent.to(torch.int64)
    ar = torch.arange(anc.numel(), device=anc.device)
    dist = (anc != ar).to(torch.int64)
    for _ in range(40):
        nxt = anc[anc]
        if torch.equal(nxt, anc):
            break
        dist = dist + dist[anc] * (anc != nxt)
        anc = nxt
    nonroot = parent.to(torch.int64) != ar
    return {"mean_depth_nonroots": round(float(dist[nonroot].double().mean()), 3)
            if bool(nonroot.any()) else 0.0, "max_depth": int(dist.max()),
            "nonroots": int(nonroot.sum())}


def filter_coverage(h, forest, n):
    """After a local run: the share of the anchor's class (vertices whose root equals the
    anchor's) already marked in the handle's R21 bitmap — the walks a bitmap-assisted
    flatten would skip."""
    from cuda.bindings import runtime as cudart
    ptr, words, anchor = h.filter_bitmap()
    if not ptr or anchor < 0:
        return None
    nw = (n + 31) // 32
    bits = torch.empty(nw, dtype=torch.int32, device="cuda")
    cudart.cudaMemcpy(bits.data_ptr(), ptr, nw * 4, cudart.cudaMemcpyKind.cudaMemcpyDeviceToDevice)
    f = forest.clone()
    h.finalize(f)
    ar = torch.arange(n, device="cuda")
    b = ((bits.to(torch.int64)[ar // 32] >> (ar % 32)) & 1).bool()
    cls = f == f[anchor]
    nonroot = f != ar
    return {"anchor_class": int(cls.sum()), "marked": int((b & cls).sum()),
            "marked_outside_class": int((b & ~cls).sum()),
            "coverage": round(float((b & cls).sum()) / max(int(cls.sum()), 1), 4),
            "nonroots": int(nonroot.sum()),
            "nonroots_outside_class": int((nonroot & ~cls).sum())}


def tree_merge(h, forests, G, n, args, ref, t_rank):
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
    fins = {}
    f = forests[0].clone()
    fins["fini3"], _ = timed(lambda: h.finalize(f), reps=1)
    del f
    h.finalize(forests[0])
    t_fin = min(fins.values())
    torch.cuda.synchronize()
    ok = bool(torch.equal(forests[0], ref))
    t_rounds = sum(max(x["round_ms"] for x in v) for v in rounds.values())
    return {"merge_rounds": rounds, "final_flatten_ms": round(t_fin, 4),
            "final_flatten_variants_ms": {k: round(v, 4) for k, v in fins.items()},
            "merge_total_ms": round(t_rounds + t_fin, 4), "labels_exact": ok,
            "projected_ms": round(max(t_rank) + t_rounds + t_fin, 4)}


def snapshot_filter(h, n):
    """Copy of a handle's R21 bitmap (merge_bits extends it: restore between timings)."""
    from cuda.bindings import runtime as cudart
    ptr, words, anchor = h.filter_bitmap()
    if not ptr:
        return None
    nw = (n + 31) // 32
    buf = torch.empty(nw, dtype=torch.int32, device="cuda")
    cudart.cudaMemcpy(buf.data_ptr(), ptr, nw * 4, cudart.cudaMemcpyKind.cudaMemcpyDeviceToDevice)
    return ptr, buf


def restore_filter(snap):
    from cuda.bindings import runtime as cudart
    if snap is not None:
        ptr, buf = snap
        cudart.cudaMemcpy(ptr, buf.data_ptr(), buf.numel() * 4,
                          cudart.cudaMemcpyKind.cudaMemcpyDeviceToDevice)


def encoded_merge(hs, forests, G, n, bounds, nidx64, args, ref, t_rank, use_filter):
    """dist.EncodedMerge on one GPU: ranks g > 0 encode their unflattened local forest
    (ECL_CC_OPT_MERGE_FILTER: with their own run's R21 bitmap as membership proofs), rank 0
    merges all encodings into its own local forest and flattens."""
    for h in hs:
        h.set_option("merge_filter", 1 if use_filter else 0)
    encs, t_enc, pair_counts = [], [], []
    for r in range(1, G):
        idx = nidx64[bounds[r]:bounds[r + 1] + 1]
        anchor = edist.row_anchor(idx, bounds[r])
        enc = hs[r].encode_buffers(n)
        t, _ = timed(lambda: hs[r].forest_encode(forests[r], anchor, enc))
        t_enc.append(t)
        pair_counts.append(int(enc["meta"][0]))
        encs.append(enc)
    h0 = hs[0]
    base = forests[0].clone()
    snap = snapshot_filter(h0, n) if use_filter else None
    f = forests[0]

    def mrg():
        f.copy_(base)
        restore_filter(snap)
        h0.merge_encoded(f, encs)
        h0.finalize(f)
    copy_t, _ = timed(lambda: (f.copy_(base), restore_filter(snap)))
    t_all, _ = timed(mrg)
    f.copy_(base)
    restore_filter(snap)
    h0.merge_encoded(f, encs)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    h0.finalize(f)
    b.record()
    b.synchronize()
    t_fin = a.elapsed_time(b)
    t_m = max(t_all - copy_t - t_fin, 0.0)
    ok = bool(torch.equal(f, ref))
    f.copy_(base)
    restore_filter(snap)
    for h in hs:
        h.set_option("merge_filter", 0)
    enc_bytes = sum(((n + 31) // 32) * 4 + 16 + 8 * c for c in pair_counts)
    xfer = enc_bytes / (args.link_gbs * 1e9) * 1e3
    ready = max([t_rank[0]] + [t_rank[r] + t_enc[r - 1] for r in range(1, G)])
    p2p = ready + max(t_m, xfer) + t_fin
    compact = ready + xfer + t_m + t_fin
    return {"filter": use_filter, "encode_ms": [round(x, 4) for x in t_enc],
            "pairs": pair_counts, "encoded_bytes_total": enc_bytes,
            "merge_ms": round(t_m, 4), "transfer_ms_model": round(xfer, 4),
            "final_flatten_ms": round(t_fin, 4),
            "merge_plus_flatten_ms": round(max(t_m, xfer) + t_fin, 4),
            "encode_merge_flatten_ms": round(max(t_enc or [0]) + max(t_m, xfer) + t_fin, 4),
            "projected_ms": round(p2p, 4), "projected_compact_ms": round(compact, 4),
            "labels_exact": ok}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--gpus", default="1,2,4,8")
    ap.add_argument("--link-gbs", type=float, default=750.0)
    ap.add_argument("--chunks", type=int, default=4)
    ap.add_argument("--even", action="store_true")
    ap.add_argument("--order", type=int, default=2, help="ECL_CC_OPT_ORDER of every run")
    ap.add_argument("--merge", default="tree,encoded")
    ap.add_argument("--calibrate", type=int, default=0,
                    help="re-partition once from the measured local-forest times")
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
        forests, t_rank, cov = [], [], []
        hs = [h] + [ecl.Handle(0) for _ in range(G - 1)]     # one handle per rank
        for hh in hs:
            hh.set_option("order", args.order)
        for r in range(G):
            lo, hi = bounds[r], bounds[r + 1]
            idx, lst = edist.slice_rows(nidx64, g.nlist, lo, hi)
            par = torch.empty(n, dtype=torch.int32, device="cuda")
            t, _ = timed(lambda: hs[r].run_rows(n, lo, hi, idx, lst, parent=par,
                                                flatten=(G == 1)))
            t_rank.append(t)
            forests.append(par)
            if G > 1:
                cov.append(filter_coverage(hs[r], par, n))
            del idx, lst
        if args.calibrate and G > 1 and wts is not None:
            # one measured step re-weights the rows (dist.rebalance_weights), then the
            # local forests are rebuilt on the new partition
            t_first = list(t_rank)
            bounds = edist.partition_rows(nidx64.cpu(), G, weights=edist.rebalance_weights(
                wts, bounds, t_rank))
            del forests
            forests, t_rank = [], []
            for r in range(G):
                lo, hi = bounds[r], bounds[r + 1]
                idx, lst = edist.slice_rows(nidx64, g.nlist, lo, hi)
                par = torch.empty(n, dtype=torch.int32, device="cuda")
                t, _ = timed(lambda: hs[r].run_rows(n, lo, hi, idx, lst, parent=par,
                                                    flatten=False))
                t_rank.append(t)
                forests.append(par)
                del idx, lst
        row = {"gpus": G, "rank_forest_ms": [round(x, 4) for x in t_rank],
               "rank_forest_ms_before_calibration":
                   [round(x, 4) for x in t_first] if args.calibrate and G > 1 else None,
               "rank_entries": [int(nidx64[bounds[r + 1]] - nidx64[bounds[r]]) for r in range(G)],
               "rank_rows": [bounds[r + 1] - bounds[r] for r in range(G)],
               "rank_depth": [depth_stats(f) for f in forests] if G > 1 else None,
               "rank_filter_coverage": cov or None}
        if "tree" in args.merge and G > 1:
            tf = [f.clone() for f in forests]
            row["tree"] = tree_merge(h, tf, G, n, args, ref, t_rank)
            del tf
        if "encoded" in args.merge and G > 1:
            row["encoded"] = encoded_merge(hs, forests, G, n, bounds, nidx64, args, ref,
                                           t_rank, False)
            row["encoded_filter"] = encoded_merge(hs, forests, G, n, bounds, nidx64, args,
                                                  ref, t_rank, True)
        if G == 1:
            row["projected_ms"] = round(t_rank[0], 4)
        best = min([row[k]["projected_ms"] for k in ("tree", "encoded", "encoded_filter")
                    if k in row] or
                   [row.get("projected_ms", t_rank[0])])
        row["projected_speedup_best"] = round(t1 / best, 3)
        res["rows"].append(row)
        del forests
        for hh in hs[1:]:
            hh.close()
        torch.cuda.empty_cache()
    print(json.dumps(res))


if __name__ == "__main__":
    main()

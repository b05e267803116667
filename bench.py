#!/usr/bin/env python
"""ECL-CC on B200: Medges/s (device-timed) and % of HBM roofline, with the CPU oracle beside.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--impl ours|reference]

One "step" = one full ECL-CC run (init_bin, depth_probe + prejump, hook_thread, hook_warp,
hook_block, finalize)
over the resident CSR of the workload (BASELINE.json configs; default C5 = Graph500
Kronecker scale 27, edge factor 16, the config the metric's 1/2/4/8-GPU figure is quoted
on).  For N > 1 (torchrun, one rank per GPU over NCCL) a step is the row-partitioned run
(ecl_cc_run_rows) plus the binomial-tree forest merge, labels on rank 0 (strong scaling:
the graph is fixed).  Prints ONE JSON line on rank 0.

Metric: m / t, m = directed CSR entries (Table 2 "Edges*" convention).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as gg  # noqa: E402

CONFIG_TEXT = {
    "C1": "uniform random graph n=2^16, avg degree 4 (CSR, symmetric)",
    "C2": "2D grid 4096x4096 with 10% random edge deletions",
    "C3": "uniform random r4-2^23",
    "C4": "R-MAT scale 24 edge factor 16",
    "C5": "Kronecker/Graph500 scale 27 edge factor 16",
}
L2_BYTES = 126 * 2 ** 20
METRIC = "Medges/s (device-timed) and % of HBM roofline at 1/2/4/8 B200 vs CPU oracle"


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        pass
    # MEASURED_PEAKS.json is driver-written per pod and not always present on the box;
    # BASELINE.md records this pool's measured copy bandwidth
    return 6437.9, "measured (BASELINE.md §2: MEASURED_PEAKS.json hbm_gbs = 6437.9 on this pool)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.3)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *exc):
        self.lines = []
        if self.proc is not None:
            time.sleep(0.1)
            self.proc.terminate()
            try:
                out, _ = self.proc.communicate(timeout=5)
            except Exception:
                self.proc.kill()
                out = ""
            self.lines = [ln for ln in out.splitlines() if ln.strip()]

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in getattr(self, "lines", []):
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for nm, val in zip(names, f[2:6]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": mx, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def build_graph(name: str, seed: int, device, scale_down: int = 0):
    t0 = time.time()
    g = gg.make_config(name, seed=seed, device=device, scale_down=scale_down)
    torch.cuda.synchronize() if str(device).startswith("cuda") else None
    return g, time.time() - t0


def algorithmic_bytes(g, parent_init, hw, lazy=False):
    """Per-kernel split of B_alg = S_idx(n+1) + 4m + 4n: every
    byte of B_alg is charged to exactly ONE kernel, so the parts sum to B_alg.
      init_bin     nindex (S_idx per offset) + the entries of every row no hook kernel
                   reads (Init3 roots — init scans their whole row, R3 — and the
                   thread-bin rows of <= 4 entries whose smaller entries all equal the
                   Init parent, R24 — init holds their whole row in registers)
      hook_thread  4 B per entry of the active thread-bin rows with hook work (R24)
      hook_warp    4 B per entry of the worklist-front rows (17..352)
      hook_block   4 B per entry of the worklist-back rows (> 352)
      finalize     4 B per label written
    With R28 (lazy: Init3 folded into the hook kernels) init_bin reads only nindex and the
    hook kernels read every entry of the rows of their degree range.
    parent_init = Init3 parents (a stop_after=1 run) on the device."""
    n, m = g.n, g.m
    s_idx = g.nindex.element_size()
    deg = g.degrees()
    dev = g.nindex.device
    v = torch.arange(n, device=dev, dtype=torch.int64)
    par = parent_init.to(torch.int64)
    active = par != v
    t1, t2 = hw
    thr = active & (deg <= t1)
    fr = active & (deg > t1) & (deg <= t2)
    bk = active & (deg > t2)
    # R24: a thread-bin row of <= 4 entries needs hook work only if it has a smaller entry
    # other than its Init parent (rows of 5..16 entries are all treated as work)
    small = thr & (deg <= 4)
    other = torch.zeros(n, dtype=torch.bool, device=dev)
    starts = g.nindex[:-1].to(torch.int64)
    for j in range(4):
        sel = small & (deg > j)
        x = g.nlist[starts[sel] + j].to(torch.int64)
        other[sel] = other[sel] | ((x < v[sel]) & (x != par[sel]))
    tw = thr & (~small | other)
    if lazy:            # R28: every non-empty row is streamed by the kernel of its bin
        nz = deg > 0
        thr, tw = nz & (deg <= t1), nz & (deg <= t1)
        fr = (deg > t1) & (deg <= t2)
        bk = deg > t2
    e_thr, e_fr, e_bk = (int(deg[x].sum()) for x in (tw, fr, bk))
    b = {
        "init_bin": s_idx * (n + 1) + 4 * (m - e_thr - e_fr - e_bk),
        "hook_thread": 4 * e_thr,
        "hook_warp": 4 * e_fr,
        "hook_block": 4 * e_bk,
        "finalize": 4 * n,
    }
    assert sum(b.values()) == s_idx * (n + 1) + 4 * m + 4 * n
    info = {"active": int(active.sum()), "thread_bin_vertices": int(thr.sum()),
            "thread_vertices": int(tw.sum()), "thread_entries": e_thr,
            "warp_vertices": int(fr.sum()), "warp_entries": e_fr,
            "block_vertices": int(bk.sum()), "block_entries": e_bk}
    return b, info


def flush_l2(buf):
    buf.add_(1)


def time_steps(fn, K, W, stream, flush_buf=None):
    """W untimed warm-ups, then K steps each bracketed by CUDA events on `stream`."""
    for _ in range(W):
        fn()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(K)]
    per = []
    for i in range(K):
        if flush_buf is not None:
            with torch.cuda.stream(stream):
                flush_l2(flush_buf)
        evs[i][0].record(stream)
        fn()
        evs[i][1].record(stream)
    torch.cuda.synchronize()
    for a, b in evs:
        per.append(a.elapsed_time(b))
    return per


# One bounded sample of every workload, used by BOTH oracle timings (cpu_baseline on
# rank 0 of our arm, and the reference arm): the same generator recipe with 2^-sd of the
# vertices (C5: 1/8 -> n = 2^24, m ~ 0.52e9; one O1 run ~3 s on one core).
SAMPLE_SD = {"C1": 0, "C2": 0, "C3": 0, "C4": 1, "C5": 3}


class PinnedCore:
    """Run the oracle pinned to one host core (`taskset -c 0`): the first
    core this process may use; the affinity is restored afterwards."""

    def __enter__(self):
        self.prev = os.sched_getaffinity(0)
        self.core = min(self.prev)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.prev)


def oracle_sample(config: str, seed: int):
    sd = SAMPLE_SD[config]
    g, _ = build_graph(config, seed, "cuda" if torch.cuda.is_available() else "cpu", sd)
    nidx, nl = g.numpy()
    del g
    return sd, nidx, nl


def sample_text(config, sd, nidx, nl, core):
    return (f"{config} recipe at 1/2^{sd} scale (n={nidx.shape[0] - 1}, m={int(nl.shape[0])}), "
            f"O1 serial BFS, pinned to host core {core} of {os.cpu_count()}")


def cpu_oracle_sample(config: str, seed: int, budget_s: float = 15.0):
    """Time the oracle (O1 BFS, 1 thread pinned to one core) on the bounded sample of the
    workload (SAMPLE_SD), repeated up to 5 times within the budget."""
    import oracle
    sd, nidx, nl = oracle_sample(config, seed)
    oracle.build()
    with PinnedCore() as pc:
        t0 = time.perf_counter()
        oracle.bfs(nidx, nl)
        dt = time.perf_counter() - t0
        reps = 1
        while dt * (reps + 1) / reps < budget_s and reps < 5:
            t1 = time.perf_counter()
            oracle.bfs(nidx, nl)
            dt += time.perf_counter() - t1
            reps += 1
    m = int(nl.shape[0])
    out = {"value": round(m * reps / dt / 1e6, 3), "unit": "Medges/s", "cores": 1,
           "kind": "oracle",
           "sample": sample_text(config, sd, nidx, nl, pc.core) + f", {reps} run(s), {dt:.2f} s"}
    return out, (nidx, nl)


def cpu_paper_codes(nidx, nl, budget_s: float = 10.0):
    """The paper's own CPU versions (ECL-CCOMP on all host cores, ECL-CCSER on one; P:L183,
    P:L185; baselines/) on the same bounded sample as cpu_baseline: context, not the
    oracle."""
    import baselines
    baselines.build()
    m = int(nl.shape[0])
    res = {}
    for name, fn, cores in (("ecl_cc_omp", lambda: baselines.omp(nidx, nl), os.cpu_count()),
                            ("ecl_cc_ser", lambda: baselines.ser(nidx, nl), 1)):
        fn()
        t0 = time.perf_counter()
        reps = 0
        while True:
            fn()
            reps += 1
            if time.perf_counter() - t0 > budget_s / 4 or reps >= 5:
                break
        dt = time.perf_counter() - t0
        res[name] = {"value": round(m * reps / dt / 1e6, 3), "unit": "Medges/s",
                     "cores": cores, "runs": reps}
    return res


def run_reference(args):
    """Reference arm = the CPU oracle as it stands (O1, one pinned core) on the bounded
    sample of the workload (SAMPLE_SD, the same sample as our arm's cpu_baseline); under
    torchrun only rank 0 runs and prints, the other ranks exit without work."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle
    sd, nidx, nl = oracle_sample(args.config, args.seed)
    oracle.build()
    with PinnedCore() as pc:
        for _ in range(args.warmup):
            oracle.bfs(nidx, nl)
        per = []
        for _ in range(args.steps):
            t0 = time.perf_counter()
            oracle.bfs(nidx, nl)
            per.append(time.perf_counter() - t0)
    m = int(nl.shape[0])
    tot = sum(per)
    value = m * args.steps / tot / 1e6
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 3), "unit": "Medges/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1e3 * tot / args.steps, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": {"workload": args.config, "description": CONFIG_TEXT[args.config],
                   "sample_scale_down": sd, "n": int(nidx.shape[0] - 1), "m": m},
        "cpu_baseline": {"value": round(value, 3), "unit": "Medges/s", "cores": 1,
                         "kind": "oracle", "sample": sample_text(args.config, sd, nidx, nl,
                                                                 pc.core)},
        "e2e": {"value": round(value, 3), "unit": "Medges/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def relaunch_with_torchrun(n: int) -> int:
    """`bench.py --gpus N` without a torchrun environment: launch the N ranks ourselves
    (one process per GPU, the driver's own launch line) and return their exit code."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={n}", "--master-addr=127.0.0.1", f"--master-port={port}",
           os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def check_world(args) -> None:
    """Run here only if the world matches --gpus: without a torchrun environment and
    N > 1, launch the N ranks ourselves (and exit with their code), or fail loudly when
    the node has fewer than N GPUs; under torchrun, WORLD_SIZE must equal N."""
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        have = torch.cuda.device_count()
        if have < args.gpus:
            print(f"bench.py: --gpus {args.gpus} needs {args.gpus} GPUs, this node has {have}",
                  file=sys.stderr)
            sys.exit(2)
        sys.exit(relaunch_with_torchrun(args.gpus))
    _, world, _ = dist_env()
    if world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}", file=sys.stderr)
        sys.exit(2)


def launches_per_step(world: int, rank: int, chunks: int, merge: str, probe: int = 0) -> int:
    """Our kernels per step on `rank`: init_bin, depth_probe, prejump (exits at once on
    shallow forests), hook_thread, hook_range x2, finalize (+ `probe`: R28's locality
    probe, launched when m < 16n); with G ranks: identity_outside
    instead of finalize in run_rows, then for the tree merge one merge_hook per received
    chunk and rank 0's finalize; for the encoded merges encode on every rank g > 0, and
    merge_bits + merge_pairs + finalize on rank 0."""
    if world == 1:
        return 7 + probe
    from paper_conf_hpdc_jaiganeshb18_b200 import dist as edist
    if merge != "tree":
        return 7 + (3 if rank == 0 else 1)
    recv = sum(1 for (_, _s, r) in edist.tree_schedule(world) if r == rank)
    return 7 + recv * chunks + (1 if rank == 0 else 0)


def launches_per_run(info: dict, world: int, rank: int, chunks: int, merge: str,
                     probe: int = 0) -> int:
    """Our kernels per timed step: ONE when the run took the R33 single-launch path
    (info["single_launch"], from ecl_cc_get_run_info), else launches_per_step."""
    if world == 1 and info.get("single_launch"):
        return 1
    return launches_per_step(world, rank, chunks, merge, probe)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C5", choices=sorted(CONFIG_TEXT))
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--load-mode", type=int, default=1)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--chunks", type=int, default=4, help="tree merge: chunks per round")
    ap.add_argument("--calibrate", type=int, default=0,
                    help="N > 1: re-partition once from measured local-forest times")
    ap.add_argument("--merge", default="p2p", choices=["p2p", "compact", "tree"],
                    help="N > 1: forest merge (dist.EncodedMerge p2p / compact, or the "
                         "binomial tree of full forests)")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--check", action="store_true", help="full oracle parity of the bench run")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    check_world(args)

    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    import paper_conf_hpdc_jaiganeshb18_b200 as ecl
    if world > 1:
        import torch.distributed as tdist
        from paper_conf_hpdc_jaiganeshb18_b200 import dist as edist
        tdist.init_process_group("nccl", device_id=dev)

    g, gen_s = build_graph(args.config, args.seed, dev)
    n, m = g.n, g.m
    s_idx = g.nindex.element_size()
    idx_dtype = str(g.nindex.dtype).replace("torch.", "")
    h = ecl.Handle(local)
    h.set_option("load_mode", args.load_mode)
    stream = torch.cuda.current_stream(dev)
    labels = torch.empty(n, dtype=torch.int32, device=dev)
    flush_buf = None if (m * 4 > 2 * L2_BYTES) else torch.zeros(64 * 2 ** 20, dtype=torch.int32,
                                                                  device=dev)
    b_alg = s_idx * (n + 1) + 4 * m + 4 * n

    # ---- algorithmic-bytes bookkeeping (outside the timed region; N=1 path) ----
    alg, info = {}, {}
    if world == 1:
        h.run(g.nindex, g.nlist, out=labels)
        run_info = h.run_info()                 # the library's own R28 / R23 decisions
        lazy = 1 if run_info["lazy_init3"] else 0
        h.set_option("stop_after", 1)
        h.run(g.nindex, g.nlist, out=labels)
        h.set_option("stop_after", 0)
        alg, info = algorithmic_bytes(g, labels, (16, 352), lazy=lazy)
        info["init"] = "R28: Init3 in the hook kernels" if lazy else "separate Init3 pass"
        info["r23_passes"] = run_info["deep_forest_passes"]
        info["r21_filter"] = run_info["filter"]
        info["single_launch"] = run_info["fused"]   # R33: the whole path in one kernel

    if world == 1:
        step = lambda: h.run(g.nindex, g.nlist, out=labels)  # noqa: E731
    else:
        # rows split by estimated work (probed entries + a streaming share); every rank
        # keeps ONLY its slice resident (the full graph is built once to cut it, outside
        # the timed region, and released)
        wts = edist.row_weights(g.nindex, g.nlist)
        bounds = edist.partition_rows(g.nindex, world, weights=wts)
        calib = None
        if args.calibrate:
            # one measured local forest per rank re-weights the rows (setup, untimed)
            lo, hi = bounds[rank], bounds[rank + 1]
            i0, l0 = edist.slice_rows(g.nindex, g.nlist, lo, hi)
            ts = []
            for _ in range(3):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                h.run_rows(n, lo, hi, i0, l0, parent=labels, flatten=False)
                e1.record(stream)
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
            t = torch.tensor([min(ts)], dtype=torch.float64, device=dev)
            allt = [torch.zeros_like(t) for _ in range(world)]
            tdist.all_gather(allt, t)
            calib = [round(float(x.item()), 4) for x in allt]
            bounds = edist.partition_rows(g.nindex, world,
                                          weights=edist.rebalance_weights(wts, bounds, calib))
            del i0, l0
        lo, hi = bounds[rank], bounds[rank + 1]
        idx_r, lst_r = edist.slice_rows(g.nindex, g.nlist, lo, hi)
        idx_r, lst_r = idx_r.clone(), lst_r.clone()
        del g
        torch.cuda.empty_cache()
        slice_entries = int(lst_r.numel())
        merger = None
        if args.merge != "tree":
            merger = edist.EncodedMerge(h, n, edist.row_anchor(idx_r, lo), mode=args.merge)

        def merge(parent):
            if merger is None:
                edist.forest_merge(parent, h, chunks=args.chunks)
            else:
                merger(parent)

        def step():
            merge(h.run_rows(n, lo, hi, idx_r, lst_r, parent=labels, flatten=False))

    # ---- timed region ----
    merger = merger if world > 1 else None
    if world > 1:
        tdist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        per = time_steps(step, args.steps, max(args.warmup, 3), stream, flush_buf)
        if world > 1:
            tdist.barrier()
        torch.cuda.synchronize()
    tot_ms = sum(per)
    if world > 1:
        t = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        tot_ms = float(t.item())
    ms_step = tot_ms / args.steps
    value = m / (ms_step * 1e-3) / 1e6

    # ---- per-phase times (separate, event-instrumented runs; N=1 path) ----
    phase, phase_seq = {}, {}
    if world == 1:
        h.set_option("timing", 1)
        reps = max(3, min(args.steps, 10))

        def phases(order):
            # per-kernel spans from the library's events + the run's own span
            h.set_option("order", order)
            acc = {k: 0.0 for k in ecl.PHASES}
            run_ms = 0.0
            for _ in range(reps):
                if flush_buf is not None:
                    flush_l2(flush_buf)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                h.run(g.nindex, g.nlist, out=labels)
                e1.record(stream)
                for k, v in h.timing().items():
                    acc[k] += v
                e1.synchronize()
                run_ms += e0.elapsed_time(e1)
            return {k: v / reps for k, v in acc.items()}, run_ms / reps

        # the paper's sequential order: each kernel alone on the GPU (matches ncu's
        # serialised launch list); then the library default (order 2: hook_block on a side
        # stream concurrent with hook_thread -> hook_warp), whose hook kernels overlap
        phase_seq, _ = phases(0)
        phase, run_ms = phases(2)
        h.set_option("timing", 0)
        hooks_ms = run_ms - phase["init_bin"] - phase["finalize"]

    # ---- parity of the bench output: I1/I2 invariants on the device ----
    # (with N ranks the labels are broadcast and every rank checks I1 on its own slice)
    ok = None
    if world == 1:
        ok = device_invariants(g.nindex, g.nlist, labels, 0, dev)
        if args.check:
            import oracle
            exp, ncc = oracle.bfs(*g.numpy())
            ok["oracle_exact"] = bool(np.array_equal(labels.cpu().numpy(), exp))
    else:
        tdist.broadcast(labels, src=0)
        mine = device_invariants(idx_r, lst_r, labels, lo, dev)
        flag = torch.tensor([int(mine["I1"]), int(mine["I2"])], dtype=torch.int32, device=dev)
        tdist.all_reduce(flag, op=tdist.ReduceOp.MIN)
        ok = {"I1": bool(flag[0]), "I2": bool(flag[1]), "components": mine["components"]}

    # ---- end-to-end through the public API with host buffers ----
    e2e = None
    if not args.no_e2e:
        if world == 1:
            hidx = g.nindex.cpu().pin_memory()
            hlst = g.nlist.cpu().pin_memory()
            hout = torch.empty(n, dtype=torch.int32).pin_memory()
            h.run_host(hidx, hlst, out=hout)
            ts = []
            for _ in range(args.e2e_steps):
                t0 = time.perf_counter()
                h.run_host(hidx, hlst, out=hout)
                ts.append(time.perf_counter() - t0)
            e2e_ms = 1e3 * sum(ts) / len(ts)
            h2d = int(hidx.numel() * hidx.element_size() + hlst.numel() * 4)
            del hidx, hlst, hout
        else:
            # every rank copies its slice host->device, runs its rows, merges; rank 0
            # copies the labels back (device-timed per rank, max over ranks)
            hidx = idx_r.cpu().pin_memory()
            hlst = lst_r.cpu().pin_memory()
            hout = torch.empty(n, dtype=torch.int32).pin_memory()
            didx, dlst = torch.empty_like(idx_r), torch.empty_like(lst_r)

            def e2e_step():
                didx.copy_(hidx, non_blocking=True)
                dlst.copy_(hlst, non_blocking=True)
                merge(h.run_rows(n, lo, hi, didx, dlst, parent=labels, flatten=False))
                if rank == 0:
                    hout.copy_(labels, non_blocking=True)

            pe = time_steps(e2e_step, args.e2e_steps, 1, stream)
            t = torch.tensor([sum(pe) / len(pe)], dtype=torch.float64, device=dev)
            tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
            e2e_ms = float(t.item())
            hb = torch.tensor([hidx.numel() * 8 + hlst.numel() * 4], dtype=torch.int64,
                              device=dev)
            tdist.all_reduce(hb)
            h2d = int(hb.item())
            del hidx, hlst, hout, didx, dlst
        e2e = {"value": round(m / (e2e_ms * 1e-3) / 1e6, 3), "unit": "Medges/s",
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": int(n * 4),
               "steps": args.e2e_steps, "ms_per_step": round(e2e_ms, 3)}

    if world > 1 and merger is not None:
        torch.cuda.synchronize()
        tdist.barrier()
        merger.close()
    if rank != 0:
        if world > 1:
            tdist.barrier()
            tdist.destroy_process_group()
        return

    peak, peak_src = peaks()
    roof = None
    if phase and info.get("single_launch"):
        # R33: the timed runs are ONE kernel (fused_small_kernel) doing the whole path, so
        # that kernel is the dominant (only) unit: B_alg over the step time.  phase_ms are
        # from separate event-instrumented runs of the multi-kernel path (context)
        achieved = b_alg / (ms_step * 1e-3) / 1e9
        tr = [ncu_traffic(args.config, k) for k in ("fused",)]
        roof = {"bound": "hbm", "kernel": "fused_small_kernel (whole path, one launch)",
                "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4),
                "traffic": None if None in tr else int(sum(tr)), "peak_source": peak_src,
                "alg_bytes_per_launch": int(b_alg), "ms_per_launch": round(ms_step, 4),
                "path_alg_bytes": int(b_alg),
                "path_frac": round(b_alg / (ms_step * 1e-3) / 1e9 / peak, 4),
                "alg_bytes_by_kernel": alg,
                "phase_ms_note": "phase_ms: separate timed runs of the multi-kernel path"}
    elif phase:
        # the three hook kernels run concurrently (order 2), so the dominant unit is the
        # concurrent hook group: the bytes of B_alg charged to them (algorithmic_bytes: the
        # entries of the rows they stream) over the span from init's end to the join (run
        # span minus init and finalize); per-kernel spans overlap
        hk = ("hook_thread", "hook_warp", "hook_block")
        alg_h = sum(alg[k] for k in hk)
        assert alg_h <= b_alg
        achieved = alg_h / (hooks_ms * 1e-3) / 1e9
        tr = [ncu_traffic(args.config, k) for k in hk]
        roof = {"bound": "hbm", "kernel": "hook_thread+hook_warp||hook_block (concurrent)",
                "achieved": round(achieved, 1),
                "peak": peak, "unit": "GB/s", "frac": round(achieved / peak, 4),
                "traffic": None if None in tr else int(sum(tr)), "peak_source": peak_src,
                "alg_bytes_per_launch": int(alg_h), "ms_per_launch": round(hooks_ms, 4),
                "path_alg_bytes": int(b_alg),
                "path_frac": round(b_alg / (ms_step * 1e-3) / 1e9 / peak, 4),
                "alg_bytes_by_kernel": alg,
                "l2_probe_ceiling": l2_probe_ceiling(info, hk, hooks_ms)}
        dom = max(phase_seq, key=phase_seq.get)
        a_seq = alg[dom] / (phase_seq[dom] * 1e-3) / 1e9
        roof["sequential_dominant"] = {
            "kernel": dom, "ms_per_launch": round(phase_seq[dom], 4),
            "achieved": round(a_seq, 1), "frac": round(a_seq / peak, 4),
            "traffic": ncu_traffic(args.config, dom),
            "l2_probe_ceiling": l2_probe_ceiling(info, (dom,), phase_seq[dom])}
    elif world > 1:
        # whole-job roofline: B_alg over the max-over-ranks step time and N x peak (SURVEY
        # §8(d) multi-GPU figure)
        roof = {"bound": "hbm", "kernel": "whole step (run_rows + forest merge)",
                "achieved": round(b_alg / (ms_step * 1e-3) / 1e9, 1), "peak": peak * world,
                "unit": "GB/s", "frac": round(b_alg / (ms_step * 1e-3) / 1e9 / (peak * world), 4),
                "traffic": None, "peak_source": peak_src + f" x {world} GPUs",
                "path_alg_bytes": int(b_alg)}
    cpu = None
    cpu_paper = None
    if world == 1 and not args.no_cpu:
        cpu, sample = cpu_oracle_sample(args.config, args.seed)
        cpu_paper = cpu_paper_codes(*sample)
        del sample

    line = {
        "metric": METRIC, "value": round(value, 3), "unit": "Medges/s", "n_gpus": world,
        "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": round(ms_step, 4),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "int32", "data": "synthetic",
        "config": {"workload": args.config, "description": CONFIG_TEXT[args.config],
                   "seed": args.seed, "n": n, "m": m, "index_dtype": idx_dtype,
                   "l2": "inputs larger than L2" if flush_buf is None else
                         "L2 flushed (256 MB write) between timed steps",
                   "parallelism": f"rows{world}" if world > 1 else "single",
                   "load_mode": args.load_mode, "gen_s": round(gen_s, 1), **info,
                   **({"rank0_rows": [lo, hi], "rank0_entries": slice_entries,
                       "merge": args.merge, "merge_chunks": args.chunks,
                       "partition": "row_weights" + (" + calibrated" if calib else ""),
                       "calibration_forest_ms": calib}
                      if world > 1 else {})},
        "gpu_launches": launches_per_run(info, world, rank, args.chunks, args.merge,
                                         probe=int(m < 16 * n)) * args.steps,
        "clocks": clk.summary(),
        "roofline": roof,
        "phase_ms": {k: round(v, 4) for k, v in phase.items()},
        "phase_ms_sequential": {k: round(v, 4) for k, v in phase_seq.items()},
        "cpu_baseline": cpu,
        "cpu_paper_codes": cpu_paper,
        "e2e": e2e,
        "parity": ok,
        "per_step_ms": [round(x, 4) for x in per],
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        tdist.barrier()
        tdist.destroy_process_group()


def device_invariants(nindex, nlist, labels, row_lo, dev, chunk=1 << 28):
    """I1 (both endpoints of every entry of rows [row_lo, row_lo + len(nindex) - 1) share a
    label) and I2 (label[v] <= v, labels are fixed points) on the device."""
    lab = labels.to(torch.int64)
    nidx64 = nindex.to(torch.int64)
    m = int(nlist.numel())
    i1 = True
    for a in range(0, m, chunk):
        pos = torch.arange(a, min(m, a + chunk), device=dev, dtype=torch.int64)
        rows = torch.searchsorted(nidx64, pos, right=True) - 1 + row_lo
        i1 &= bool((lab[rows] == lab[nlist[a:a + chunk].to(torch.int64)]).all())
        del pos, rows
    ar = torch.arange(lab.numel(), device=dev)
    i2 = bool((lab <= ar).all()) and bool((lab[lab] == lab).all())
    return {"I1": i1, "I2": i2, "components": int((lab == ar).sum())}


def l2_probe_ceiling(info, kernel, ms):
    """The binding resource of the hook kernels is L2 requests, one per probed edge
    (DESIGN.md §5).  Compare the kernel with the measured ceiling of exactly that access
    pattern (tools/l2_ceiling.py: stream the adjacency, probe one bitmap word for every
    other entry, nothing else; profiles/l2_ceiling.json)."""
    keys = {"hook_block": "block_entries", "hook_warp": "warp_entries",
            "hook_thread": "thread_entries"}
    if isinstance(kernel, str):
        kernel = (kernel,)
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "l2_ceiling.json")))
        rate = float(d["probe_pattern_entries_G_s"]) * 1e9
    except Exception:
        return None
    if any(k not in keys for k in kernel):
        return None
    entries = sum(int(info.get(keys[k]) or 0) for k in kernel)
    if not entries:
        return None
    t_ceil = entries / rate * 1e3
    return {"entries": entries, "ceiling_entries_G_s": rate / 1e9,
            "ms_at_ceiling": round(t_ceil, 4), "frac": round(t_ceil / ms, 4),
            "source": "profiles/l2_ceiling.json (tools/l2_ceiling.py probe pattern)"}


def ncu_traffic(config, kernel):
    """DRAM bytes per launch of `kernel` from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        d = json.load(open(p))
        return d[config][kernel]
    except Exception:
        return None


if __name__ == "__main__":
    main()

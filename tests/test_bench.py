"""bench.py contract pieces that run without a GPU: the reference arm (the CPU oracle on a
bounded sample, task contract ④) and the roofline bookkeeping helpers."""
import json
import os
import subprocess
import sys

import numpy as np
import torch

import bench
import graphgen as gg
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_prints_one_contract_line():
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--steps", "2", "--warmup", "1", "--config", "C1"],
                         capture_output=True, text=True, env=env, timeout=600, check=True).stdout
    lines = [ln for ln in out.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["unit"] == "Medges/s" and d["value"] > 0
    assert d["steps"] == 2 and d["warmup"] == 1 and d["higher_is_better"] is True
    assert d["config"]["workload"] == "C1"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"] == {"value": d["value"], "unit": "Medges/s", "h2d_bytes_per_step": 0,
                        "d2h_bytes_per_step": 0}


def test_reference_arm_other_ranks_are_silent():
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="", RANK="1", WORLD_SIZE="2")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--steps", "1", "--warmup", "0", "--config", "C1"],
                         capture_output=True, text=True, env=env, timeout=600, check=True).stdout
    assert not [ln for ln in out.splitlines() if ln.startswith("{")]


def test_algorithmic_bytes_partition_b_alg():
    """The per-kernel parts sum to B_alg = S_idx(n+1) + 4m + 4n; bins follow
    R2/R3 and the thread-bin work rows follow R24, checked against a plain loop."""
    for name, sd in (("C4", 8), ("C1", 2), ("C2", 8)):
        g = gg.shuffle_rows(gg.make_config(name, seed=3, scale_down=sd), seed=1)
        nidx, nl = g.numpy()
        init3 = oracle.init3(nidx, nl)
        alg, info = bench.algorithmic_bytes(g, torch.from_numpy(init3), (16, 352))
        s_idx = g.nindex.element_size()
        assert sum(alg.values()) == s_idx * (g.n + 1) + 4 * g.m + 4 * g.n
        assert alg["finalize"] == 4 * g.n and all(x >= 0 for x in alg.values())
        e = {"thread": 0, "warp": 0, "block": 0}
        nv = {"thread": 0, "warp": 0, "block": 0}
        for v in range(g.n):
            row = nl[nidx[v]:nidx[v + 1]]
            p = init3[v]
            if p == v:
                continue
            d = len(row)
            if d <= 16:
                if d <= 4 and not any(x < v and x != p for x in row):
                    continue
                k = "thread"
            else:
                k = "warp" if d <= 352 else "block"
            e[k] += d
            nv[k] += 1
        for k in e:
            assert info[f"{k}_entries"] == e[k] and info[f"{k}_vertices"] == nv[k], (name, k)
        assert info["active"] == int((init3 != np.arange(g.n)).sum())
        lz, li = bench.algorithmic_bytes(g, torch.from_numpy(init3), (16, 352), lazy=1)
        assert sum(lz.values()) == sum(alg.values())
        assert lz["init_bin"] == s_idx * (g.n + 1)          # R28: only nindex
        deg = np.diff(nidx.astype(np.int64))
        assert li["thread_entries"] == int(deg[deg <= 16].sum())
        assert li["block_entries"] == int(deg[deg > 352].sum())


def test_l2_probe_ceiling_uses_the_committed_measurement():
    r = bench.l2_probe_ceiling({"block_entries": 526_200_000}, "hook_block", 2.0)
    assert r is not None and abs(r["ms_at_ceiling"] - 1.0) < 1e-3 and abs(r["frac"] - 0.5) < 1e-3
    assert bench.l2_probe_ceiling({}, "finalize", 1.0) is None


def test_l2_probe_ceiling_of_the_concurrent_hook_group():
    # order 2 runs the three hook kernels concurrently: the ceiling covers their entries
    info = {"thread_entries": 100_000_000, "warp_entries": 200_000_000,
            "block_entries": 226_200_000}
    r = bench.l2_probe_ceiling(info, ("hook_thread", "hook_warp", "hook_block"), 2.0)
    assert r["entries"] == 526_200_000
    assert abs(r["ms_at_ceiling"] - 1.0) < 1e-3 and abs(r["frac"] - 0.5) < 1e-3
    assert bench.l2_probe_ceiling(info, ("hook_block", "finalize"), 1.0) is None


def test_gpus_flag_fails_without_enough_gpus():
    """`bench.py --gpus 2` without a torchrun environment launches 2 ranks itself, and
    fails loudly (no silent 1-rank line) on a node with fewer GPUs."""
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2",
                        "--steps", "1", "--config", "C1"], capture_output=True, text=True,
                       env=env, timeout=300)
    assert r.returncode != 0 and "needs 2 GPUs" in r.stderr
    assert not [ln for ln in r.stdout.splitlines() if ln.startswith("{")]


def test_gpus_flag_must_match_world():
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="", WORLD_SIZE="3", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2",
                        "--steps", "1", "--config", "C1"], capture_output=True, text=True,
                       env=env, timeout=300)
    assert r.returncode != 0 and "WORLD_SIZE=3" in r.stderr


def test_single_launch_counts_one_kernel_per_step():
    # R33: a run that took the single-launch path is ONE kernel (fused_small_kernel);
    # the multi-kernel count applies otherwise
    import bench
    assert bench.launches_per_run({"single_launch": True}, 1, 0, 4, "p2p", probe=1) == 1
    assert bench.launches_per_run({"single_launch": False}, 1, 0, 4, "p2p") == 7
    assert bench.launches_per_run({}, 1, 0, 4, "p2p", probe=1) == 8
    assert bench.launches_per_run({"single_launch": True}, 2, 0, 4, "p2p") == \
        bench.launches_per_step(2, 0, 4, "p2p")

"""bench.py contract pieces that run without a GPU: the reference arm (the CPU oracle on a
bounded sample, task contract ④) and the roofline bookkeeping helpers."""
import json
import os
import subprocess
import sys

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


def test_algorithmic_bytes_partition_the_rows():
    """Per-bin entries add up to the entries of active rows, bins follow R2/R3."""
    g = gg.make_config("C4", seed=3, scale_down=8)
    nidx, nl = g.numpy()
    init3 = torch.from_numpy(oracle.init3(nidx, nl))
    alg, info = bench.algorithmic_bytes(g, init3, (16, 352))
    deg = g.degrees()
    active = init3.to(torch.int64) != torch.arange(g.n)
    assert info["active"] == int(active.sum())
    assert (info["thread_entries"] + info["warp_entries"] + info["block_entries"]
            == int(deg[active].sum()))
    assert info["thread_vertices"] == int((active & (deg <= 16)).sum())
    assert info["block_vertices"] == int((active & (deg > 352)).sum())
    assert alg["finalize"] == 8 * g.n
    assert all(v >= 0 for v in alg.values())


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

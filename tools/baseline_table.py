"""BASELINE.md §4 'Measured' table from the committed bench lines and ncu traffic logs.

    python tools/baseline_table.py profiles/r2/final   # bench_C{1..5}.json, traffic_C{1..5}.csv

Per config: Medges/s (bench value), the path's % of the HBM roofline (B_alg / t over 8 TB/s
nominal and over the measured copy peak), ncu DRAM GB/s and L2 hit rate over all of our
kernels of one run (bytes / summed kernel durations; sector-weighted hit rate), the oracle
(O1, one pinned core) seconds on its sample, and the parity status.
"""
import csv
import json
import os
import sys
from collections import defaultdict


def bench(d, c):
    p = os.path.join(d, f"bench_{c}.json")
    if not os.path.exists(p):
        return None
    return json.loads(open(p).read().strip().splitlines()[-1])


def traffic(d, c):
    p = os.path.join(d, f"traffic_{c}.csv")
    if not os.path.exists(p):
        return None
    rows = [r for r in csv.reader(open(p)) if len(r) > 12 and r[0] != "ID"]
    per = defaultdict(dict)
    for r in rows:
        try:
            per[(r[0], r[4])][r[12]] = float(r[14].replace(",", ""))
        except (ValueError, IndexError):
            pass
    dram = sum(m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
               for m in per.values())
    dur = sum(m.get("gpu__time_duration.sum", 0) for m in per.values())   # ns
    sect = sum(m.get("lts__t_sectors.sum", 0) for m in per.values())
    hits = sum(m.get("lts__t_sectors.sum", 0) * m.get("lts__t_sector_hit_rate.pct", 0) / 100
               for m in per.values())
    return {"dram_gbs": dram / dur if dur else None, "l2_hit": 100 * hits / sect if sect else None,
            "dram_gb": dram / 1e9, "kernels_ms": dur / 1e6}


def main(d):
    names = {"C1": "C1 ER 2^16", "C2": "C2 grid 4096², 10 % deleted", "C3": "C3 r4-2^23",
             "C4": "C4 R-MAT s24 ef16", "C5": "C5 Graph500 s27 ef16"}
    print("| Config | GPUs | ms / run | Medges/s | % of HBM roofline (8 TB/s / measured) | "
          "ncu DRAM GB/s | L2 hit % | Oracle O1 (1 pinned core) | Parity |")
    print("|---|---|---:|---:|---:|---:|---:|---|---|")
    for c in ("C1", "C2", "C3", "C4", "C5"):
        b = bench(d, c)
        if b is None:
            continue
        t = traffic(d, c)
        r = b["roofline"]
        balg = r["path_alg_bytes"]
        s = b["ms_per_step"] * 1e-3
        nom, meas = balg / s / 8e12, r["path_frac"]
        cpu = b.get("cpu_baseline") or {}
        samp = cpu.get("sample", "")
        m_s = samp.split("m=")[1].split(")")[0] if "m=" in samp else None
        osec = f"{int(m_s) / (cpu['value'] * 1e6):.2f} s on {samp.split(' (')[0]}" if m_s else "—"
        par = b.get("parity") or {}
        ok = "I1/I2 hold on the bench output; bit-exact vs O1 at full size (tests)" \
            if par.get("I1") and par.get("I2") else "FAIL"
        print(f"| {names[c]} | 1 | {b['ms_per_step']:.4f} | {b['value']:,.0f} | "
              f"{100 * nom:.1f} % / {100 * meas:.1f} % | "
              f"{t['dram_gbs']:.0f} | {t['l2_hit']:.1f} | {osec} | {ok} |"
              if t else
              f"| {names[c]} | 1 | {b['ms_per_step']:.4f} | {b['value']:,.0f} | "
              f"{100 * nom:.1f} % / {100 * meas:.1f} % | — | — | {osec} | {ok} |")


if __name__ == "__main__":
    main(sys.argv[1])

"""Turn ncu --csv metric logs into per-kernel tables (profiles/*.md, profiles/*.json)."""
import csv
import io
import json
import re
import sys

NAMES = {"init_bin": "init_bin", "hook_thread": "hook_thread", "ILi16ELb1": "hook_warp",
         "16, true": "hook_warp", "16, 1": "hook_warp", "64, false": "hook_block",
         "64, 0": "hook_block", "finalize": "finalize"}


def kname(s):
    if "init_bin" in s:
        return "init_bin"
    if "hook_thread" in s:
        return "hook_thread"
    if "hook_range" in s:
        return "hook_warp" if re.search(r"16,\s*(1|true)", s) else "hook_block"
    if "finalize" in s:
        return "finalize"
    if "locality_probe" in s:
        return "locality_probe"
    if "fused_small" in s:
        return "fused"
    if "prejump" in s:
        return "prejump"
    if "depth_probe" in s:
        return "depth_probe"
    return s[:40]


def load(path):
    txt = open(path).read()
    lines = [ln for ln in txt.splitlines() if ln.startswith('"')]
    rows = list(csv.DictReader(io.StringIO("\n".join(lines))))
    per = {}
    for r in rows:
        k = (r["ID"], kname(r["Kernel Name"]))
        per.setdefault(k, {})[r["Metric Name"]] = (float(r["Metric Value"].replace(",", "")),
                                                     r["Metric Unit"])
    return per


if __name__ == "__main__":
    out = {}
    for path in sys.argv[1:]:
        per = load(path)
        print(f"\n{path}")
        for (i, k), m in sorted(per.items(), key=lambda kv: int(kv[0][0])):
            print(f"  #{i:>3} {k:12s} " + "  ".join(f"{n.split('.')[0]}={v:.4g}{u}" for n, (v, u) in sorted(m.items())))

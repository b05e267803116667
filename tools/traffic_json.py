"""Build profiles/ncu_traffic.json (DRAM read+write bytes per launch, per config and kernel)
from ncu --metrics logs written by tools/gpu_profile.sh.

    python tools/traffic_json.py TAG   # reads gpurun_out/TAG_traffic_C{1..5}.csv
    python tools/traffic_json.py DIR   # reads DIR/traffic_C{1..5}.csv (tools/gpu_final.sh)
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_tables import load  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main(tag):
    out = {}
    for c in ("C1", "C2", "C3", "C4", "C5"):
        path = os.path.join(ROOT, "gpurun_out", f"{tag}_traffic_{c}.csv")
        if os.path.isdir(tag):                  # tools/gpu_final.sh layout: DIR/traffic_Cn.csv
            path = os.path.join(tag, f"traffic_{c}.csv")
        if not os.path.exists(path):
            continue
        per = load(path)
        out[c] = {}
        for (_, k), m in sorted(per.items(), key=lambda kv: int(kv[0][0])):
            b = m["dram__bytes_read.sum"][0] + m["dram__bytes_write.sum"][0]
            out[c][k] = int(b)
    out["_source"] = (f"ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum "
                      f"--clock-control none, one run per config (tools/gpu_profile.sh, tag {tag})")
    with open(os.path.join(ROOT, "profiles", "ncu_traffic.json"), "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "prof")

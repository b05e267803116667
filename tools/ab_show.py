"""Print the per-phase table of a gpurun_out/ab_<tag>.jsonl file (tools/ab_run.sh)."""
import json
import re
import sys

txt = open(sys.argv[1]).read()
for blob in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try:
        d = json.loads(blob.replace("\n", " "))
    except json.JSONDecodeError:
        print("unparsable:", blob[:120].replace("\n", " "))
        continue
    r = d["r"]
    b = r["best_ms"]
    print(f"{r['config']} {d['variant']:12s} total={b['total']:7.3f} init={b['init_bin']:.3f} "
          f"thr={b['hook_thread']:.3f} warp={b['hook_warp']:.3f} blk={b['hook_block']:.3f} "
          f"fin={b['finalize']:.3f}")

#!/bin/bash
# Round-2 GPU call AB: R31 quads in hook_warp only (vec 2, new default) vs both (1) vs none (0).
O=gpurun_out/r2ab; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests/test_gpu_vec.py tests/test_gpu_fused.py -x -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for c in C4 C5; do for o in 2 0; do for v in 2 1 0 2 1 0 2 1 0; do timeout 300 python tools/prof.py --config $c --reps 10 --vec $v --order $o; done; done; done > $O/ab_vec.jsonl 2>&1
python -c "
import json, statistics as st
r={}
for l in open('$O/ab_vec.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); b=d['best_ms']; r.setdefault((d['config'], d['order'], d['vec']), []).append((b['total'], b['hook_warp'], b['hook_block']))
for k in sorted(r): print(k, 'total', [x[0] for x in r[k]], 'warp', [x[1] for x in r[k]], 'block', [x[2] for x in r[k]])"

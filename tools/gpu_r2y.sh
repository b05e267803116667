#!/bin/bash
# Round-2 GPU call Y: R31 quads auto-on for int32 offsets (vec 2) vs off; fused grid = SMs.
O=gpurun_out/r2y; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests/test_gpu_vec.py tests/test_gpu_fused.py -x -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for c in C2 C3 C4 C5; do for v in 2 0 2 0 2 0; do timeout 300 python tools/prof.py --config $c --reps 10 --vec $v; done; done > $O/ab_vec_auto.jsonl 2>&1
python -c "
import json
for l in open('$O/ab_vec_auto.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); b=d['best_ms']; print(d['config'], 'vec', d['vec'], 'thr %.3f warp %.3f block %.3f total %.3f' % (b['hook_thread'], b['hook_warp'], b['hook_block'], b['total']))"
for spec in "C1 0" "C2 6" "C3 5" "C4 7" "C5 11"; do
  set -- $spec
  for f in 0 1 0 1; do timeout 300 python tools/prof.py --config $1 --scale-down $2 --reps 20 --timing 0 --fused $f; done
done > $O/ab_fused.jsonl 2>&1
python -c "
import json
for l in open('$O/ab_fused.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['config'], d['n'], d['m'], 'fused', d['fused'], d['best_ms'])"

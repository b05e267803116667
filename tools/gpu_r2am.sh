#!/bin/bash
# Round-2 GPU call AM: plain (unbatched) hooking vs the queue engine on single-launch graphs.
O=gpurun_out/r2am; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for spec in "C1 0" "C2 6" "C2 4" "C3 5" "C3 4" "C4 8" "C4 7" "C5 11" "C5 10"; do
  set -- $spec
  for b in 1 0 1 0 1 0; do timeout 300 python tools/prof.py --config $1 --scale-down $2 --reps 20 --timing 0 --batch $b; done
done > $O/ab_batch.jsonl 2>&1
python -c "
import json, statistics as st
r={}
for l in open('$O/ab_batch.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); r.setdefault((d['config'], d['n'], d['m'], d['fused'], d['bjif'][0]), []).append(d['best_ms']['total'])
for k in sorted(r): print(k, 'min %.4f' % min(r[k]), [round(x,4) for x in r[k]])"

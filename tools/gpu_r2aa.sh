#!/bin/bash
# Round-2 GPU call AA: R21 filter forced on vs auto on the L2-resident configs (R28 graphs).
O=gpurun_out/r2aa; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
for c in C3 C1 C2; do for f in 2 1 2 1 2 1 2 1 2 1; do timeout 300 python tools/prof.py --config $c --reps 10 --filter $f --timing 0; done; done > $O/ab_filter.jsonl 2>&1
python -c "
import json, statistics as st
r={}
for l in open('$O/ab_filter.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); r.setdefault((d['config'], d['filter']), []).append(d['best_ms']['total'])
for k in sorted(r): print(k, 'min %.4f median %.4f' % (min(r[k]), st.median(r[k])), [round(x,3) for x in r[k]])"

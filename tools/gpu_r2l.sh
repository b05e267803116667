#!/bin/bash
# Round-2 GPU call L (new session): smoke, R21 filter forced on for the L2-resident configs,
# default C5 bench line.
O=gpurun_out/r2l; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
for c in C1 C2 C3 C4; do for f in 2 1 2 1; do timeout 300 python tools/prof.py --config $c --reps 10 --filter $f; done; done > $O/ab_filter.jsonl 2>&1
python -c "
import json
for l in open('$O/ab_filter.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['config'], 'filter', d['filter'], d['best_ms'])"
timeout 600 python bench.py > $O/bench_C5.json 2> $O/bench_C5.err; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('$O/bench_C5.json').read().strip().splitlines()[-1])
print('C5', d['ms_per_step'], d['value'], d['roofline']['frac'], d['phase_ms'], d['phase_ms_sequential'], d['clocks'])"

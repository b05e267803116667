#!/bin/bash
# Round-2 GPU call Z: R23 pass grid (blocks per SM) x interleaved vertices on C2; the fused
# path's size crossover (forced on/off on 2^19-2^21-row graphs).
O=gpurun_out/r2z; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
for pass in 1 2 3; do for v in cur pj1o1 pj4o1 pj4o2 pj8o1; do
  echo -n "{\"variant\": \"$v\", \"r\": "
  ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config C2 --reps 10 2>&1 | tail -1
  echo "}"
done; done > $O/ab_pj.jsonl
python - <<'P'
import json,re
txt=open('gpurun_out/r2z/ab_pj.jsonl').read()
for blk in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try: d=json.loads(blk.replace('\n',''))
    except Exception: print(blk[:300]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], '%-6s'%d['variant'], 'init %.3f thr %.3f total %.3f' % (b['init_bin'], b['hook_thread'], b['total']))
P
for spec in "C2 5" "C2 4" "C3 4" "C3 3" "C4 6" "C4 5" "C5 10" "C5 9"; do
  set -- $spec
  for f in 0 1 0 1; do timeout 300 python tools/prof.py --config $1 --scale-down $2 --reps 20 --timing 0 --fused $f; done
done > $O/ab_fused_size.jsonl 2>&1
python -c "
import json
for l in open('$O/ab_fused_size.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['config'], d['n'], d['m'], 'fused', d['fused'], d['best_ms'])"

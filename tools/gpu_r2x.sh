#!/bin/bash
# Round-2 GPU call X: R23 passes with 4 interleaved vertices per thread; fused-path grid size.
O=gpurun_out/r2x; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests/test_gpu_fused.py tests/test_gpu_parity.py -x -q -k "prejump or fused or configs or hand" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for c in C2 C4; do
  for pass in 1 2 3; do for v in pj4 pj1 pj8; do
    echo -n "{\"variant\": \"$v\", \"r\": "
    ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config $c --reps 10 2>&1 | tail -1
    echo "}"
  done; done
done > $O/ab_pj.jsonl
python - <<'P'
import json,re
txt=open('gpurun_out/r2x/ab_pj.jsonl').read()
for blk in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try: d=json.loads(blk.replace('\n',''))
    except Exception: print(blk[:300]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], '%-5s'%d['variant'], 'init %.3f thr %.3f warp %.3f block %.3f fin %.3f total %.3f' % (b['init_bin'], b['hook_thread'], b['hook_warp'], b['hook_block'], b['finalize'], b['total']))
P
for g in 0 148 296 592; do for r in 1 2; do timeout 300 python tools/prof.py --config C1 --reps 30 --timing 0 --grid $g; done; done > $O/ab_c1_grid.jsonl 2>&1
python -c "
import json
for l in open('$O/ab_c1_grid.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print('C1 grid', d.get('grid', '?'), d['fused'], d['best_ms'])"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"prejump" -c 1 \
  -o $O/full_C2_pj python tools/prof.py --config C2 --reps 1 > /dev/null 2>&1; echo "ncu C2 rc=$?"
python tools/ncu_summary.py $O/full_C2_pj.ncu-rep > $O/full_C2_prejump.txt 2>&1
rm -f $O/*.ncu-rep
grep -i "Duration\|issued\|L2 Cache Throughput" $O/full_C2_prejump.txt

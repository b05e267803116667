#!/bin/bash
# Round-2 GPU call AG: init_bin row-prefix loads with an L2 prefetch-size hint.
O=gpurun_out/r2ag; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
for c in C5 C4 C2; do
  for pass in 1 2 3; do for v in pf0 pf64 pf128 pf256; do
    echo -n "{\"variant\": \"$v\", \"r\": "
    ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config $c --reps 10 2>&1 | tail -1
    echo "}"
  done; done
done > $O/ab_pf.jsonl
python - <<'P'
import json,re
txt=open('gpurun_out/r2ag/ab_pf.jsonl').read()
for blk in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try: d=json.loads(blk.replace('\n',''))
    except Exception: print(blk[:300]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], '%-6s'%d['variant'], 'init %.3f thr %.3f warp %.3f block %.3f fin %.3f total %.3f' % (b['init_bin'], b['hook_thread'], b['hook_warp'], b['hook_block'], b['finalize'], b['total']))
P
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for v in pf0 pf256; do
  ECL_CC_LIB=build/ab/$v.so timeout 600 ncu --metrics $M --clock-control none -k regex:"init_bin" --csv --log-file $O/traffic_init_C5_$v.csv \
    python tools/prof.py --config C5 --reps 1 > /dev/null 2>&1; echo "traffic $v rc=$?"
  python tools/ncu_tables.py $O/traffic_init_C5_$v.csv | grep -o "#.*"
done

#!/bin/bash
# Round-2 GPU call AI: R36 (a piece joins the anchor's tree when it hooks a marked u).
O=gpurun_out/r2ai; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_raw_csr.py tests/test_gpu_dist.py -x -q -k "filter or membership or C5 or raw or dist or forest" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -x -q -k "exact and C5" > $O/pytest_full.log 2>&1; echo "pytest full C5 rc=$?"; tail -2 $O/pytest_full.log
for o in 2 0; do for pass in 1 2 3; do for v in r36 nor36; do
  echo -n "{\"variant\": \"$v\", \"r\": "
  ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config C5 --reps 10 --order $o 2>&1 | tail -1
  echo "}"
done; done; done > $O/ab_r36.jsonl
python - <<'P'
import json,re
txt=open('gpurun_out/r2ai/ab_r36.jsonl').read()
for blk in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try: d=json.loads(blk.replace('\n',''))
    except Exception: print(blk[:300]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], 'order', r['order'], '%-6s'%d['variant'], 'init %.3f thr %.3f warp %.3f block %.3f fin %.3f total %.3f' % (b['init_bin'], b['hook_thread'], b['hook_warp'], b['hook_block'], b['finalize'], b['total']))
P
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for v in r36 nor36; do
  ECL_CC_LIB=build/ab/$v.so timeout 600 ncu --metrics $M --clock-control none -k regex:"hook" --csv --log-file $O/traffic_C5_$v.csv \
    python tools/prof.py --config C5 --reps 1 > /dev/null 2>&1; echo "traffic $v rc=$?"
  python tools/ncu_tables.py $O/traffic_C5_$v.csv | grep -o "#.*dram__bytes_write=[0-9.e+]*byte"
done

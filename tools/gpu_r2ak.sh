#!/bin/bash
# Round-2 GPU call AK: R21 bitmap as a persisting L2 access-policy window (hook kernels).
O=gpurun_out/r2ak; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -x -q -k "membership or filter or order or configs or stream or graph" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for pass in 1 2 3; do for v in persist np; do
  echo -n "{\"variant\": \"$v\", \"r\": "
  ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config C5 --reps 10 2>&1 | tail -1
  echo "}"
done; done > $O/ab_persist.jsonl
python - <<'P'
import json,re
txt=open('gpurun_out/r2ak/ab_persist.jsonl').read()
for blk in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try: d=json.loads(blk.replace('\n',''))
    except Exception: print(blk[:300]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], '%-8s'%d['variant'], 'init %.3f thr %.3f warp %.3f block %.3f fin %.3f total %.3f' % (b['init_bin'], b['hook_thread'], b['hook_warp'], b['hook_block'], b['finalize'], b['total']))
P
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for v in persist np; do
  ECL_CC_LIB=build/ab/$v.so timeout 600 ncu --metrics $M --clock-control none -k regex:"hook" --csv --log-file $O/traffic_C5_$v.csv \
    python tools/prof.py --config C5 --reps 1 > /dev/null 2>&1; echo "traffic $v rc=$?"
  python tools/ncu_tables.py $O/traffic_C5_$v.csv | grep -o "#.*dram__bytes_write=[0-9.e+]*byte"
done

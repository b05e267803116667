#!/bin/bash
# Round-2 GPU call AE: R35 anchor row first in hook_block — parity, A/B on C5 (orders 2/0).
O=gpurun_out/r2ae; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_raw_csr.py tests/test_gpu_fused.py tests/test_gpu_vec.py tests/test_gpu_dist.py -x -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -x -q -k "C5" > $O/pytest_full.log 2>&1; echo "pytest full C5 rc=$?"; tail -2 $O/pytest_full.log
for o in 2 0; do for pass in 1 2 3; do for v in af noaf; do
  echo -n "{\"variant\": \"$v\", \"r\": "
  ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config C5 --reps 10 --order $o 2>&1 | tail -1
  echo "}"
done; done; done > $O/ab_af.jsonl
python - <<'P'
import json,re
txt=open('gpurun_out/r2ae/ab_af.jsonl').read()
for blk in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try: d=json.loads(blk.replace('\n',''))
    except Exception: print(blk[:300]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], 'order', r['order'], '%-5s'%d['variant'], 'init %.3f thr %.3f warp %.3f block %.3f fin %.3f total %.3f' % (b['init_bin'], b['hook_thread'], b['hook_warp'], b['hook_block'], b['finalize'], b['total']))
P
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
K='regex:hook|init_bin|finalize'
for v in af noaf; do
  ECL_CC_LIB=build/ab/$v.so timeout 600 ncu --metrics $M --clock-control none -k "$K" --csv --log-file $O/traffic_C5_$v.csv \
    python tools/prof.py --config C5 --reps 1 > /dev/null 2>&1; echo "traffic $v rc=$?"
  python tools/ncu_tables.py $O/traffic_C5_$v.csv | grep -o "#.*dram__bytes_write=[0-9.e+]*byte"
done

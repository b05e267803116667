#!/bin/bash
# Round-2 GPU call V: R34 deferred v_rep walk in hook_thread — parity, A/B vs not deferring.
O=gpurun_out/r2v; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_raw_csr.py tests/test_gpu_fused.py -x -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for c in C1 C2 C3 C4 C5; do
  for pass in 1 2 3; do for v in defer nodefer; do
    echo -n "{\"variant\": \"$v\", \"r\": "
    ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config $c --reps 10 2>&1 | tail -1
    echo "}"
  done; done
done > $O/ab_defer.jsonl
python - <<'P'
import json,re
txt=open('gpurun_out/r2v/ab_defer.jsonl').read()
for blk in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try: d=json.loads(blk.replace('\n',''))
    except Exception: print(blk[:300]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], '%-8s'%d['variant'], 'init %.3f thr %.3f warp %.3f block %.3f fin %.3f total %.3f' % (b['init_bin'], b['hook_thread'], b['hook_warp'], b['hook_block'], b['finalize'], b['total']))
P

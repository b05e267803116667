#!/bin/bash
# Round-2 GPU call O: R32 carried queue — parity, A/B carry / nocarry / minb6 on C1..C5.
O=gpurun_out/r2s; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 900 python -m pytest tests/test_gpu_vec.py tests/test_gpu_raw_csr.py -x -q > $O/pytest_vec.log 2>&1; echo "pytest vec/raw rc=$?"; tail -1 $O/pytest_vec.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "configs_scaled or hand_built or forest or membership or order_ or ablation or stats" > $O/pytest_par.log 2>&1; echo "pytest par rc=$?"; tail -1 $O/pytest_par.log
for c in C1 C2 C3 C4 C5; do
  for pass in 1 2 3; do for v in smallq bigq; do
    echo -n "{\"variant\": \"$v\", \"r\": "
    ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config $c --reps 10 2>&1 | tail -1
    echo "}"
  done; done
done > $O/ab_carry.jsonl
python - <<'P'
import json,re
txt=open('gpurun_out/r2s/ab_carry.jsonl').read()
for blk in re.findall(r'\{"variant".*?\n\}', txt, re.S):
    try: d=json.loads(blk.replace('\n',''))
    except Exception: print(blk[:300]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], '%-8s'%d['variant'], 'init %.3f thr %.3f warp %.3f block %.3f fin %.3f total %.3f' % (b['init_bin'], b['hook_thread'], b['hook_warp'], b['hook_block'], b['finalize'], b['total']))
P

#!/bin/bash
# Round-2 GPU call N: lean quad engine A/B (vec 0/1) x register caps / quads per round.
O=gpurun_out/r2n; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_vec.py -x -q > $O/pytest_vec.log 2>&1; echo "pytest vec rc=$?"; tail -1 $O/pytest_vec.log
for c in C4 C5; do
  for spec in base@--vec=0 base minb6 vq2 minb6vq2 minb5 minb6@--vec=0 base@--vec=0 base minb6; do
    for o in 0 2; do
      v=${spec%%@*}; a=""; [[ "$spec" == *@* ]] && a=${spec#*@}
      echo -n "{\"variant\": \"$spec\", \"order\": $o, \"r\": "
      ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config $c --reps 6 --order $o ${a//,/ } 2>&1 | tail -1
      echo "}"
    done
  done
done > $O/ab_quads.jsonl
python - <<'P'
import json
for l in open('gpurun_out/r2n/ab_quads.jsonl'):
    try: d=json.loads(l)
    except Exception: print(l[:200]); continue
    r=d['r']; b=r['best_ms']
    print(r['config'], d['variant'], 'order', d['order'], 'thr %.3f warp %.3f block %.3f total %.3f' % (b['hook_thread'], b['hook_warp'], b['hook_block'], b['total']))
P

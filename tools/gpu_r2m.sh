#!/bin/bash
# Round-2 GPU call M: R31 quad engine — parity, A/B vec 0/1, ncu of the C5 range kernels.
O=gpurun_out/r2m; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 900 python -m pytest tests/test_gpu_vec.py -x -q > $O/pytest_vec.log 2>&1; echo "pytest vec rc=$?"; tail -3 $O/pytest_vec.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "configs_scaled or hand_built or forest or membership or order_ or raw" > $O/pytest_par.log 2>&1; echo "pytest par rc=$?"; tail -3 $O/pytest_par.log
for c in C4 C5; do for o in 0 2; do for v in 0 1 0 1; do timeout 300 python tools/prof.py --config $c --reps 8 --vec $v --order $o; done; done; done > $O/ab_vec.jsonl 2>&1
python -c "
import json
for l in open('$O/ab_vec.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['config'], 'order', d['order'], 'vec', d['vec'], d['best_ms'])"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hook_range" -c 2 \
  -o $O/full_C5_range python tools/prof.py --config C5 --reps 1 --order 0 > /dev/null 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $O/full_C5_range.ncu-rep > $O/full_C5_range.txt 2>&1
python tools/ncu_lines.py $O/full_C5_range.ncu-rep "(int)16, (bool)1" 40 > $O/full_C5_hook_warp_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5_range.ncu-rep "(int)64, (bool)0" 40 > $O/full_C5_hook_block_lines.txt 2>&1
grep -i "instructions\|issued\|Throughput\|dram__bytes" $O/full_C5_range.txt | head -20
rm -f $O/*.ncu-rep

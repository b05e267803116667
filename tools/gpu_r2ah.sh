#!/bin/bash
# Round-2 GPU call AH: the paper ablations (Figs. 7/8/9, Table 4) at the final defaults.
O=gpurun_out/r2ah; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1800 python tools/ablation.py C1 C2 C3 C4 > $O/ablation.jsonl 2> $O/ablation.err; echo "ablation rc=$?"
timeout 1500 python tools/ablation.py --skip Jump3 C5 >> $O/ablation.jsonl 2>> $O/ablation.err; echo "ablation C5 rc=$?"
tail -3 $O/ablation.err
wc -l $O/ablation.jsonl

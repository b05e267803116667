#!/bin/bash
# Round-2 GPU call F: init_bin offset prefetch x R28 modes (0 separate pass, 3 range rows
# lazy, 1 all rows lazy); full GPU suite.
O=gpurun_out/r2f; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
bash tools/ab_run.sh pf_fuse "C2 C3 C4 C5" pf0@--fuse=0 pf1@--fuse=0 pf1@--fuse=3 pf1@--fuse=1 pf0@--fuse=0 pf1@--fuse=0 pf1@--fuse=3 pf1@--fuse=1 > /dev/null 2>&1
mv gpurun_out/ab_pf_fuse.jsonl $O/; python tools/ab_show.py $O/ab_pf_fuse.jsonl
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log

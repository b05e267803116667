#!/bin/bash
# Round-2 GPU call AL: the full GPU suite + smoke + C5 bench at the final tree.
O=gpurun_out/r2al; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench_C5.json 2> $O/bench_C5.err; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('$O/bench_C5.json').read().strip().splitlines()[-1])
print('C5', d['ms_per_step'], d['value'], d['roofline']['frac'], d['e2e']['value'], d['gpu_launches'], d['clocks'])"

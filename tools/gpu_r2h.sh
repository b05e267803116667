#!/bin/bash
# Round-2 GPU call H: R28 auto (device locality probe); GPU suite; bench C1..C5; emulation
# with anchor-bitmap coverage.
O=gpurun_out/r2h; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
for c in C1 C2 C3; do for f in 0 2 0 2; do timeout 300 python tools/prof.py --config $c --reps 10 --fuse $f; done; done > $O/ab_fuse_auto.jsonl 2>&1
cut -c1-300 $O/ab_fuse_auto.jsonl
for c in C1 C2 C3 C4 C5; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "bench $c rc=$?"; done
for c in C1 C2 C3 C4 C5; do python -c "
import json; d=json.loads(open('$O/bench_$c.json').read().strip().splitlines()[-1])
print('$c', d['ms_per_step'], d['value'], d['roofline']['frac'], d['config'].get('init'), d['clocks'])"; done
timeout 900 python tools/mgpu_emulate.py --config C5 --gpus 2,4,8 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"

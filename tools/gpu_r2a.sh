#!/bin/bash
# Round-2 GPU call A: full GPU test suite, bench lines for C1..C5, sanitizers.
mkdir -p gpurun_out/r2a
O=gpurun_out/r2a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench_C5.json 2> $O/bench_C5.err; echo "bench C5 rc=$?"
for c in C1 C2 C3 C4; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "bench $c rc=$?"; done
timeout 300 python bench.py --gpus 2 --config C1 > $O/bench_gpus2.out 2>&1; echo "bench --gpus 2 rc=$? (must be non-zero on 1 GPU)"
for t in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_cases.py --quick > $O/sanitizer_$t.log 2>&1; echo "$t rc=$?"
  tail -3 $O/sanitizer_$t.log
done

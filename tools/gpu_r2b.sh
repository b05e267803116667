#!/bin/bash
# Round-2 GPU call B: new tests (encoded merge, multi-process), racecheck after the R18
# atomics, C5 multi-GPU emulation with both merges.
O=gpurun_out/r2b; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python -m pytest tests/test_gpu_dist.py tests/test_gpu_parity.py -m gpu -x -q -k "encode or multiprocess or ablation or forest" > $O/pytest_new.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_new.log
timeout 1500 compute-sanitizer --tool racecheck --print-limit 50 python tools/sanitize_cases.py --quick --variants > $O/sanitizer_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -3 $O/sanitizer_racecheck.log
timeout 900 python tools/mgpu_emulate.py --config C5 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"
timeout 600 python tools/mgpu_emulate.py --config C4 > $O/mgpu_emulation_C4.json 2>> $O/mgpu.err; echo "emulate C4 rc=$?"
for c in C2 C3 C4 C5; do timeout 300 python tools/prof.py --config $c --reps 10; done > $O/prof.jsonl 2>&1; cat $O/prof.jsonl

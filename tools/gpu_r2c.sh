#!/bin/bash
# Round-2 GPU call C: new tests, racecheck incl. ablation paths, owner-search A/B,
# multi-GPU emulation with flatten variants, ablations (Figs. 7-9, Table 4).
O=gpurun_out/r2c; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_raw_csr.py -m gpu -x -q -k "flatten or path_length or encode or multi_gpu or hand or configs" > $O/pytest_new.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_new.log
timeout 1500 compute-sanitizer --tool racecheck --print-limit 50 python tools/sanitize_cases.py --quick --variants > $O/sanitizer_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -3 $O/sanitizer_racecheck.log
bash tools/ab_run.sh owner "C1 C2 C3 C4 C5" walk shfl walk_qg4 shfl_qg4 > /dev/null 2>&1; cp gpurun_out/ab_owner.jsonl $O/
python tools/ab_show.py $O/ab_owner.jsonl 2>/dev/null | head -40
timeout 900 python tools/mgpu_emulate.py --config C5 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"
timeout 600 python tools/mgpu_emulate.py --config C4 > $O/mgpu_emulation_C4.json 2>> $O/mgpu.err; echo "emulate C4 rc=$?"
timeout 1200 python tools/ablation.py C1 C2 C3 C4 > $O/ablation.jsonl 2> $O/ablation.err; echo "ablation rc=$?"
timeout 900 python tools/ablation.py --skip Jump3 C5 >> $O/ablation.jsonl 2>> $O/ablation.err; echo "ablation C5 rc=$?"
cat $O/ablation.jsonl | cut -c1-400

#!/bin/bash
# Round-2 GPU call G: init_bin block-range mode, R29 sub-warp rows, R23 pass tuning;
# racecheck, GPU suite, ncu of the new hook_warp.
O=gpurun_out/r2g; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
bash tools/ab_run.sh brsw "C3 C4 C5" base0 br sw both both_qg2 both_m6 base0 both > /dev/null 2>&1
mv gpurun_out/ab_brsw.jsonl $O/; python tools/ab_show.py $O/ab_brsw.jsonl
bash tools/ab_run.sh pass "C2" both ph6 ps16 ph6ps16 both ph6 ps16 ph6ps16 > /dev/null 2>&1
mv gpurun_out/ab_pass.jsonl $O/; python tools/ab_show.py $O/ab_pass.jsonl
bash tools/ab_run.sh fuse "C1 C3 C4" both@--fuse=0 both@--fuse=1 both@--fuse=3 both@--fuse=0 both@--fuse=1 both@--fuse=3 > /dev/null 2>&1
mv gpurun_out/ab_fuse.jsonl $O/; python tools/ab_show.py $O/ab_fuse.jsonl
for v in base0 both; do ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config C5 --reps 5 --order 0; done > $O/order0.jsonl 2>&1; cut -c1-330 $O/order0.jsonl
timeout 1200 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_cases.py --quick > $O/sanitizer_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -2 $O/sanitizer_racecheck.log
timeout 1200 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_cases.py --quick > $O/sanitizer_memcheck.log 2>&1; echo "memcheck rc=$?"; tail -2 $O/sanitizer_memcheck.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hook_range|init_bin" -c 3 \
  -o $O/full_C5 python tools/prof.py --config C5 --reps 1 --order 0 > /dev/null 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $O/full_C5.ncu-rep > $O/full_C5.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "16, (bool)1" 50 > $O/full_C5_hook_warp_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "init_bin" 40 > $O/full_C5_init_lines.txt 2>&1
rm -f $O/*.ncu-rep; du -sh $O

mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "prejump or configs_scaled or hand_built or chain" > gpurun_out/pj_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pj_pytest.log
for c in C1 C2 C3 C4 C5; do for pj in 0 2; do timeout 300 python tools/prof.py --config $c --reps 10 --prejump $pj 2>&1 | tail -1; done; done > gpurun_out/pj_prof.jsonl
cat gpurun_out/pj_prof.jsonl | cut -c150-400
bash tools/ab_run.sh hops "C2" h1 h2 h3 h5 | cut -c1-30,200-500

mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err; echo "bench rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"hook_range" -c 1 -o gpurun_out/u1_full_C4_hook_warp python tools/prof.py --config C4 --reps 1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hook_range" -s 1 -c 1 -o gpurun_out/u1_full_C5_hook_block python tools/prof.py --config C5 --reps 1 > /dev/null 2>&1
ls gpurun_out

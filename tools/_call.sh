mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/l2_ceiling.py > gpurun_out/l2_ceiling.json 2>&1; cat gpurun_out/l2_ceiling.json
timeout 600 python bench.py > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err; echo "bench rc=$?"
bash tools/gpu_profile.sh r1c > gpurun_out/r1c_profile.log 2>&1

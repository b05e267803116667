#!/bin/bash
# One GPU call's worth of profiling evidence (run under gpurun from the repo root):
#   stats counters, per-kernel DRAM/L2 traffic for C1..C5, the bench launch list, and
#   ncu --set full captures of the C5 dominant kernel and the C2 hook kernel.
# Usage: bash tools/gpu_profile.sh [TAG]   -> gpurun_out/<TAG>_*
set -x
mkdir -p gpurun_out
TAG=${1:-prof}
python -c "import __graft_entry__ as g; g.build()"
for c in C1 C2 C3 C4 C5; do timeout 300 python tools/prof.py --config $c --reps 3 --stats; done > gpurun_out/${TAG}_stats.jsonl 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__t_sectors_op_atom.sum,lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum
for c in C1 C2 C3 C4 C5; do
  timeout 600 ncu --metrics $M --clock-control none -k regex:"init_bin|prejump|hook|finalize" --csv \
    --log-file gpurun_out/${TAG}_traffic_$c.csv python tools/prof.py --config $c --reps 1 > /dev/null 2>&1
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"init_bin|probe|prejump|hook|finalize" \
  --csv --log-file gpurun_out/${TAG}_launches_C5_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e > gpurun_out/${TAG}_bench_under_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hook_range" -c 2 \
  -o gpurun_out/${TAG}_full_C5_hook_range python tools/prof.py --config C5 --reps 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"hook_thread" -c 1 \
  -o gpurun_out/${TAG}_full_C2_hook_thread python tools/prof.py --config C2 --reps 1 > /dev/null 2>&1
ls -la gpurun_out

#!/bin/bash
# Round-2 evidence run T (current code): GPU suite, smoke, bench lines C1..C5 + reference
# arm, the bench's ncu launch list, per-kernel traffic C1..C5, ncu --set full of the C5
# hook kernels + init and of hook_thread on C1 / C3, sanitizers, multi-GPU emulation.
TAG=${1:-r2t}
O=gpurun_out/$TAG; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_gpu.log
for c in C5 C1 C2 C3 C4; do timeout 900 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "bench $c rc=$?"; done
for c in C1 C2 C3 C4 C5; do python -c "
import json; d=json.loads(open('$O/bench_$c.json').read().strip().splitlines()[-1])
print('$c', d['ms_per_step'], d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks'])"; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference_C5.json 2>&1; echo "reference rc=$?"
K='regex:locality|init_bin|depth_probe|prejump|hook|finalize'
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" --csv \
  --log-file $O/launches_C5_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e > $O/bench_under_ncu.log 2>&1; echo "launches rc=$?"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_atom.sum
for c in C1 C2 C3 C4 C5; do
  timeout 600 ncu --metrics $M --clock-control none -k "$K" --csv --log-file $O/traffic_$c.csv \
    python tools/prof.py --config $c --reps 1 > /dev/null 2>&1; echo "traffic $c rc=$?"
done
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"hook_range|hook_thread|init_bin" -c 4 \
  -o $O/full_C5 python tools/prof.py --config C5 --reps 1 --order 0 > /dev/null 2>&1; echo "ncu full C5 rc=$?"
python tools/ncu_summary.py $O/full_C5.ncu-rep > $O/full_C5.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "64, (bool)0" 40 > $O/full_C5_hook_block_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "16, (bool)1" 40 > $O/full_C5_hook_warp_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "hook_thread" 40 > $O/full_C5_hook_thread_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "init_bin" 40 > $O/full_C5_init_lines.txt 2>&1
for c in C1 C3; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"hook_thread" -c 1 \
    -o $O/full_${c}_thread python tools/prof.py --config $c --reps 1 > /dev/null 2>&1; echo "ncu $c rc=$?"
  python tools/ncu_summary.py $O/full_${c}_thread.ncu-rep > $O/full_${c}_hook_thread.txt 2>&1
  python tools/ncu_lines.py $O/full_${c}_thread.ncu-rep "hook_thread" 50 > $O/full_${c}_hook_thread_lines.txt 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"prejump|init_bin" -c 2 \
  -o $O/full_C2_init python tools/prof.py --config C2 --reps 1 > /dev/null 2>&1; echo "ncu C2 init rc=$?"
python tools/ncu_summary.py $O/full_C2_init.ncu-rep > $O/full_C2_init_prejump.txt 2>&1
python tools/ncu_lines.py $O/full_C2_init.ncu-rep "prejump" 30 > $O/full_C2_prejump_lines.txt 2>&1
rm -f $O/*.ncu-rep
for t in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_cases.py --quick --variants > $O/sanitizer_$t.log 2>&1; echo "$t rc=$?"; tail -2 $O/sanitizer_$t.log
done
timeout 1500 python tools/mgpu_emulate.py --config C5 --gpus 2,4,8 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"
du -sh $O

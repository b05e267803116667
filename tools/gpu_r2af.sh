#!/bin/bash
# Round-2 GPU call AF: final bench lines (after R35), reference arm, C5 launch list + traffic.
O=gpurun_out/r2af; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
for c in C5 C1 C2 C3 C4; do timeout 900 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "bench $c rc=$?"; done
for c in C1 C2 C3 C4 C5; do python -c "
import json; d=json.loads(open('$O/bench_$c.json').read().strip().splitlines()[-1])
print('$c', d['ms_per_step'], d['value'], d['roofline']['frac'], d['e2e']['value'], d['gpu_launches'], d['clocks'])"; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference_C5.json 2>&1; echo "reference rc=$?"
K='regex:fused|locality|init_bin|depth_probe|prejump|hook|finalize'
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_atom.sum
for c in C1 C2 C3 C4 C5; do
  timeout 600 ncu --metrics $M --clock-control none -k "$K" --csv --log-file $O/traffic_$c.csv \
    python tools/prof.py --config $c --reps 1 > /dev/null 2>&1; echo "traffic $c rc=$?"
done
timeout 600 ncu --metrics $M --clock-control none -k "$K" --csv --log-file $O/traffic_C1_fused.csv \
    python tools/prof.py --config C1 --reps 1 --timing 0 > /dev/null 2>&1; echo "traffic C1 fused rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" --csv \
  --log-file $O/launches_C5_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e > $O/bench_under_ncu.log 2>&1; echo "launches C5 rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"hook_range|hook_thread|init_bin" -c 4 \
  -o $O/full_C5 python tools/prof.py --config C5 --reps 1 --order 0 > /dev/null 2>&1; echo "ncu full C5 rc=$?"
python tools/ncu_summary.py $O/full_C5.ncu-rep > $O/full_C5.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "64, (bool)0" 40 > $O/full_C5_hook_block_lines.txt 2>&1
rm -f $O/*.ncu-rep
timeout 1500 python tools/mgpu_emulate.py --config C5 --gpus 2,4,8 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"

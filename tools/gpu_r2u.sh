#!/bin/bash
# Round-2 GPU call U: R33 single-launch path — parity, C1 timing fused vs multi-kernel,
# scaled graphs around the auto threshold, C1 bench line.
O=gpurun_out/r2u; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1200 python -m pytest tests/test_gpu_fused.py -x -q > $O/pytest_fused.log 2>&1; echo "pytest fused rc=$?"; tail -3 $O/pytest_fused.log
for spec in "C1 0" "C2 6" "C2 5" "C3 6" "C3 5" "C4 8" "C4 7" "C5 12" "C5 11"; do
  set -- $spec
  for f in 0 1 0 1; do timeout 300 python tools/prof.py --config $1 --scale-down $2 --reps 20 --timing 0 --fused $f; done
done > $O/ab_fused.jsonl 2>&1
python - <<'P'
import json
for l in open('gpurun_out/r2u/ab_fused.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['config'], d['n'], d['m'], 'fused', d['fused'], d['best_ms'])
P
timeout 600 python bench.py --config C1 > $O/bench_C1.json 2> $O/bench_C1.err; echo "bench C1 rc=$?"
python -c "
import json; d=json.loads(open('$O/bench_C1.json').read().strip().splitlines()[-1])
print('C1', d['ms_per_step'], d['value'], d['roofline'], d['gpu_launches'], d['config'].get('single_launch'))"
K='regex:fused|locality|init_bin|depth_probe|prejump|hook|finalize'
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_atom.sum
timeout 600 ncu --metrics $M --clock-control none -k "$K" --csv --log-file $O/traffic_C1_fused.csv \
    python tools/prof.py --config C1 --reps 1 --timing 0 > /dev/null 2>&1; echo "traffic fused rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"fused" -c 1 \
    -o $O/full_C1_fused python tools/prof.py --config C1 --reps 1 --timing 0 > /dev/null 2>&1; echo "ncu fused rc=$?"
python tools/ncu_summary.py $O/full_C1_fused.ncu-rep > $O/full_C1_fused.txt 2>&1
python tools/ncu_lines.py $O/full_C1_fused.ncu-rep "fused" 50 > $O/full_C1_fused_lines.txt 2>&1
rm -f $O/*.ncu-rep

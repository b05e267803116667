#!/bin/bash
# Round-2 GPU call AC: bench lines at the final default (R31 hook_warp quads with int32
# offsets), parity subsets, C4 traffic, R21 filter A/B on the L2-resident configs.
O=gpurun_out/r2ac; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests/test_gpu_vec.py tests/test_gpu_fused.py tests/test_gpu_parity.py tests/test_gpu_raw_csr.py -x -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
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
bash tools/gpu_r2aa.sh

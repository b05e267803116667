#!/bin/bash
# Final evidence of a round (run under gpurun from the repo root):
#   bash tools/gpu_final.sh TAG   -> gpurun_out/TAG/ (kept < 64 MiB: reports summarised, deleted)
# GPU suite, smoke, bench lines C1..C5, the bench's ncu launch list, per-kernel traffic
# C1..C5, ncu --set full of the C5 hook kernels, sanitizers, ablations (Figs. 7-9 / Table 4),
# Table 3 (L2 read/write sectors per Jump variant), multi-GPU emulation.
TAG=${1:-final}
O=gpurun_out/$TAG; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_gpu.log
for c in C5 C1 C2 C3 C4; do timeout 900 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "bench $c rc=$?"; done
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
  -o $O/full_C5 python tools/prof.py --config C5 --reps 1 --order 0 > /dev/null 2>&1; echo "ncu full rc=$?"
python tools/ncu_summary.py $O/full_C5.ncu-rep > $O/full_C5.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "64, (bool)0" 40 > $O/full_C5_hook_block_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "16, (bool)1" 40 > $O/full_C5_hook_warp_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "hook_thread" 40 > $O/full_C5_hook_thread_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5.ncu-rep "init_bin" 40 > $O/full_C5_init_lines.txt 2>&1
rm -f $O/*.ncu-rep
for t in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_cases.py --quick --variants > $O/sanitizer_$t.log 2>&1; echo "$t rc=$?"; tail -2 $O/sanitizer_$t.log
done
timeout 1500 python tools/ablation.py C1 C2 C3 C4 > $O/ablation.jsonl 2> $O/ablation.err; echo "ablation rc=$?"
timeout 1200 python tools/ablation.py --skip Jump3 C5 >> $O/ablation.jsonl 2>> $O/ablation.err; echo "ablation C5 rc=$?"
MR=lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,gpu__time_duration.sum
for c in C1 C2 C3 C4 C5; do for j in 4 1 2 3 p; do
  if [ $c = C5 ] && [ $j = 3 ]; then continue; fi
  if [ $j = p ]; then a="--jump 4 --batch 0"; else a="--jump $j"; fi
  timeout 600 ncu --metrics $MR --clock-control none -k "$K" --csv --log-file $O/l2rw_${c}_J$j.csv \
    python tools/prof.py --config $c --reps 1 $a > /dev/null 2>&1
done; done
python tools/table3.py $O > $O/table3.json; gzip -f $O/l2rw_*.csv
timeout 1500 python tools/mgpu_emulate.py --config C5 --gpus 2,4,8 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"
du -sh $O

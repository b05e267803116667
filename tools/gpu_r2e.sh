#!/bin/bash
# Round-2 GPU call E: R28 lazy Init3 — parity suite, A/B against the separate Init3 pass;
# ncu captures (summaries kept, reports deleted: gpurun_out must stay < 64 MiB); Table 3.
O=gpurun_out/r2e; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
for c in C3 C4 C5; do for f in 0 1 0 1; do timeout 300 python tools/prof.py --config $c --reps 10 --fuse $f; done; done > $O/ab_fuse.jsonl 2>&1
cut -c1-330 $O/ab_fuse.jsonl
for c in C4 C5; do for f in 0 1; do timeout 300 python tools/prof.py --config $c --reps 5 --fuse $f --order 0; done; done > $O/ab_fuse_order0.jsonl 2>&1
cut -c1-330 $O/ab_fuse_order0.jsonl
K='regex:init_bin|depth_probe|prejump|hook|finalize'
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hook_range" -c 2 \
  -o $O/full_C5_hook_range python tools/prof.py --config C5 --reps 1 --order 0 --fuse 0 > /dev/null 2>&1; echo "ncu range rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"init_bin" -c 1 \
  -o $O/full_C5_init python tools/prof.py --config C5 --reps 1 --fuse 0 > /dev/null 2>&1; echo "ncu init rc=$?"
for c in C3 C2; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"hook_thread" -c 1 \
  -o $O/full_${c}_hook_thread python tools/prof.py --config $c --reps 1 > /dev/null 2>&1; echo "ncu thread $c rc=$?"
done
for r in $O/*.ncu-rep; do python tools/ncu_summary.py $r > ${r%.ncu-rep}.txt 2>&1; python tools/ncu_lines.py $r "" 60 > ${r%.ncu-rep}_lines.txt 2>&1; done
python tools/ncu_lines.py $O/full_C5_hook_range.ncu-rep "16, (bool)1" 60 > $O/full_C5_hook_warp_lines.txt 2>&1
python tools/ncu_lines.py $O/full_C5_hook_range.ncu-rep "64, (bool)0" 60 > $O/full_C5_hook_block_lines.txt 2>&1
ncu -i $O/full_C5_hook_range.ncu-rep --page raw --csv > $O/full_C5_hook_range_raw.csv 2>/dev/null
ncu -i $O/full_C3_hook_thread.ncu-rep --page raw --csv > $O/full_C3_hook_thread_raw.csv 2>/dev/null
rm -f $O/*.ncu-rep
M=lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,gpu__time_duration.sum
for c in C1 C2 C3 C4 C5; do for j in 4 1 2 3; do
  if [ $c = C5 ] && [ $j = 3 ]; then continue; fi
  timeout 600 ncu --metrics $M --clock-control none -k "$K" --csv --log-file $O/l2rw_${c}_J$j.csv \
    python tools/prof.py --config $c --reps 1 --jump $j > /dev/null 2>&1; echo "l2rw $c J$j rc=$?"
done; done
python tools/table3.py $O > $O/table3.json; cat $O/table3.json
gzip $O/l2rw_*.csv
timeout 900 python tools/mgpu_emulate.py --config C5 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"
du -sh $O; ls -la $O

#!/bin/bash
# Round-2 GPU call D: ncu --set full captures (C5 hook_range x2, C5 init, C3/C2 hook_thread),
# Table 3 L2 read/write sectors per Jump variant (C1..C5), L2 fetch granularity A/B.
O=gpurun_out/r2d; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hook_range" -c 2 \
  -o $O/full_C5_hook_range python tools/prof.py --config C5 --reps 1 --order 0 > /dev/null 2>&1; echo "ncu range rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"init_bin" -c 1 \
  -o $O/full_C5_init python tools/prof.py --config C5 --reps 1 > /dev/null 2>&1; echo "ncu init rc=$?"
for c in C3 C2; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"hook_thread" -c 1 \
  -o $O/full_${c}_hook_thread python tools/prof.py --config $c --reps 1 > /dev/null 2>&1; echo "ncu thread $c rc=$?"
done
M=lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,lts__t_requests_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_write.sum,gpu__time_duration.sum
for c in C1 C2 C3 C4 C5; do for j in 4 1 2 3; do
  if [ $c = C5 ] && [ $j = 3 ]; then continue; fi
  timeout 600 ncu --metrics $M --clock-control none --csv --log-file $O/l2rw_${c}_J$j.csv \
    python tools/prof.py --config $c --reps 1 --jump $j > /dev/null 2>&1; echo "l2rw $c J$j rc=$?"
done; done
python tools/table3.py $O > $O/table3.json; cat $O/table3.json
for c in C3 C4 C5; do for f in 0 32; do timeout 300 python tools/prof.py --config $c --reps 10 --l2fetch $f; done; done > $O/l2fetch_ab.jsonl 2>&1
cat $O/l2fetch_ab.jsonl | cut -c1-300
for r in $O/*.ncu-rep; do python tools/ncu_summary.py $r > ${r%.ncu-rep}.txt 2>&1; python tools/ncu_lines.py $r "" 60 > ${r%.ncu-rep}_lines.txt 2>&1; done
ls -la $O
for c in C1 C2 C3 C4; do for bj in "1 4" "0 4" "0 2"; do set -- $bj; timeout 300 python tools/prof.py --config $c --reps 10 --batch $1 --jump $2; done; done > $O/plain_vs_engine.jsonl 2>&1
cut -c1-260 $O/plain_vs_engine.jsonl
timeout 900 python tools/mgpu_emulate.py --config C5 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -m gpu -x -q -k "encode or multi_gpu or flatten" > $O/pytest_merge.log 2>&1; echo "pytest merge rc=$?"; tail -2 $O/pytest_merge.log

#!/bin/bash
# Round-2 GPU call J: C3/C1 run-to-run spread vs launch options; ncu of merge_bits (8 ranks).
O=gpurun_out/r2j; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for opts in "" "order=0" "ttas=0" "load_mode=0" "occ_thread=4" "grid_blocks=148" "grid_blocks=592" "fuse_init=0 order=0" "prejump=0" ; do
  timeout 300 python tools/variance.py --config C3 --runs 25 --opt $opts
done > $O/variance_C3_opts.jsonl 2>&1
python -c "
import json
for l in open('$O/variance_C3_opts.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print('C3', d['opts'], d['min'], d['median'], d['max'])"
for opts in "" "order=0" "grid_blocks=74" "grid_blocks=148" "occ_thread=2" "fuse_init=0"; do
  timeout 300 python tools/variance.py --config C1 --runs 25 --opt $opts
done > $O/variance_C1_opts.jsonl 2>&1
python -c "
import json
for l in open('$O/variance_C1_opts.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print('C1', d['opts'], d['min'], d['median'], d['max'])"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"merge_bits|encode_kernel|finalize_filter" -c 3 \
  -o $O/full_merge python tools/mgpu_emulate.py --config C5 --gpus 8 --merge encoded > /dev/null 2>&1; echo "ncu merge rc=$?"
python tools/ncu_summary.py $O/full_merge.ncu-rep > $O/full_merge.txt 2>&1
python tools/ncu_lines.py $O/full_merge.ncu-rep "merge_bits" 40 > $O/full_merge_bits_lines.txt 2>&1
rm -f $O/*.ncu-rep; du -sh $O

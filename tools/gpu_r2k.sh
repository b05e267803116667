#!/bin/bash
O=gpurun_out/r2k; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"merge_bits" -s 4 -c 1 \
  -o $O/merge_filter python tools/mgpu_emulate.py --config C5 --gpus 8 --merge encoded > /dev/null 2>&1; echo "ncu merge rc=$?"
python tools/ncu_summary.py $O/merge_filter.ncu-rep > $O/merge_filter.txt 2>&1
python tools/ncu_lines.py $O/merge_filter.ncu-rep "merge_bits" 40 > $O/merge_filter_lines.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"finalize_filter|encode_kernel" -s 7 -c 2 \
  -o $O/enc_fin python tools/mgpu_emulate.py --config C5 --gpus 8 --merge encoded > /dev/null 2>&1; echo "ncu enc rc=$?"
python tools/ncu_summary.py $O/enc_fin.ncu-rep > $O/enc_fin.txt 2>&1
rm -f $O/*.ncu-rep; du -sh $O

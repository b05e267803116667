#!/bin/bash
# Round-2 GPU call AJ: where hook_block's DRAM traffic comes from (concurrent order: under
# ncu the kernels serialise in launch order, hook_block first) — per-source-line memory
# columns of the ncu source page.
O=gpurun_out/r2aj; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"hook_range" -c 1 \
  -o $O/full_C5_block_first python tools/prof.py --config C5 --reps 1 --order 2 > /dev/null 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $O/full_C5_block_first.ncu-rep > $O/full_C5_block_first.txt 2>&1
ncu -i $O/full_C5_block_first.ncu-rep --page source --csv --print-source cuda,sass > $O/source.csv 2>&1; echo "source rc=$?"
python - <<'P' > gpurun_out/r2aj/source_columns.txt 2>&1
import csv, io
txt = open('gpurun_out/r2aj/source.csv').read()
rows = list(csv.reader(io.StringIO(txt)))
hdr = next(r for r in rows if r and r[0] == "Line No")
print(hdr)
P
gzip -f $O/source.csv
rm -f $O/*.ncu-rep
ls -la $O

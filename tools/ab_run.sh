#!/bin/bash
# Run tools/prof.py over build/ab/*.so variants (dev A/B) -> gpurun_out/ab_<tag>.jsonl
#   bash tools/ab_run.sh TAG "C2 C3 C4 C5" [variant[@prof args] ...]
# e.g.  base  base@--order=1  pf256@--order=1
mkdir -p gpurun_out
TAG=$1; CFGS=$2; shift 2
VARS=${@:-$(cd build/ab && ls *.so | sed 's/\.so$//')}
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for c in $CFGS; do
  for spec in $VARS; do
    v=${spec%%@*}; a=""
    [[ "$spec" == *@* ]] && a=${spec#*@}
    echo -n "{\"variant\": \"$spec\", \"r\": "
    ECL_CC_LIB=build/ab/$v.so timeout 300 python tools/prof.py --config $c --reps 10 ${a//,/ } 2>&1 | tail -1
    echo "}"
  done
done > gpurun_out/ab_$TAG.jsonl
cat gpurun_out/ab_$TAG.jsonl

#!/bin/bash
# dev cycle on the GPU box: build, GPU parity tests (optionally filtered), A/B of build/ab/*.so
#   bash tools/ab_cycle.sh TAG "CONFIGS" "PYTEST_K" [variants...]
mkdir -p gpurun_out
TAG=$1; CFGS=$2; K=$3; shift 3
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
if [ -n "$K" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"
  tail -3 gpurun_out/${TAG}_pytest.log
fi
bash tools/ab_run.sh $TAG "$CFGS" "$@" > /dev/null 2>&1
python tools/ab_show.py gpurun_out/ab_$TAG.jsonl

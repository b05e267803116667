#!/bin/bash
# Round-2 GPU call I: filter-assisted encoded merge (tests + emulation), C3 spread, QG8.
O=gpurun_out/r2i; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -m gpu -x -q -k "encode or multi_gpu or multiprocess or fuse or flatten" > $O/pytest_merge.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_merge.log
timeout 1200 python tools/mgpu_emulate.py --config C5 --gpus 2,4,8 > $O/mgpu_emulation_C5.json 2> $O/mgpu.err; echo "emulate rc=$?"; tail -3 $O/mgpu.err
for f in 0 2; do timeout 300 python tools/variance.py --config C3 --runs 30 --opt fuse_init=$f; done > $O/variance_C3.jsonl 2>&1; cut -c1-400 $O/variance_C3.jsonl
timeout 300 python tools/variance.py --config C3 --runs 15 --stats > $O/variance_C3_stats.jsonl 2>&1; cut -c1-1500 $O/variance_C3_stats.jsonl
bash tools/ab_run.sh qg "C2 C3 C5" qg4 qg8 qg8m6 qg4 qg8 qg8m6 > /dev/null 2>&1
mv gpurun_out/ab_qg.jsonl $O/; python tools/ab_show.py $O/ab_qg.jsonl

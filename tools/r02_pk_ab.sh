#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_packed_gpu.py tests/test_peer_exchange_gpu.py -q -x -p no:cacheprovider --timeout 300 2>&1 | tail -2
for nb in 0 1; do
if [ $nb = 1 ]; then export FP_PK_NOBANK=1; fi
timeout 300 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('nobank=$nb ms', d['ms_per_step'], d['roofline']['frac'], d['config']['packed_copy'])"
done
unset FP_PK_NOBANK
timeout 900 ncu --set full --clock-control none --import-source on -k k_pk -c 1 -o gpurun_out/pk_c4_full -f python bench.py --config C4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > gpurun_out/pk_ncu.log 2>&1

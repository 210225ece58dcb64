#!/bin/bash
# k_pk1 ring: packed tests, then C3 / S3 timings over block size and ring depth
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x 2>&1 | tail -4
for c in C3 S3; do
for bs in 512 768 1024; do
for ns in 0 2 3 4; do
FP_PK_BS1=$bs FP_PK1_NS=$ns timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$c bs=$bs ns=$ns ms', d['ms_per_step'], d['roofline']['frac'])" 2>/dev/null
done; done; done

#!/bin/bash
# k_pk1 ring with v in the slot: packed tests, then C3 / S3 timings over ring depth
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x -k "packed1 or packed_integer" 2>&1 | tail -2
for c in C3 S3; do
for ns in 0 1 2 3; do
FP_PK1_NS=$ns timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$c ns=$ns ms', d['ms_per_step'], d['roofline']['frac'])" 2>/dev/null
done; done

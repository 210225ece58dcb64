#!/bin/bash
cd $GRAFT_REPO_ROOT
FP_PK_ROWS=32 FP_PK_SPAN=512 timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x -k "packed_ and not packed1" 2>&1 | tail -1
for rs in "64 1024" "32 1024" "64 512" "32 512" "16 512"; do
set -- $rs
FP_PK_ROWS=$1 FP_PK_SPAN=$2 timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4 rows=$1 span=$2', d['ms_per_step'], d['roofline']['frac'], d['config']['packed_copy']['tiles'])"
done

#!/bin/bash
cd $GRAFT_REPO_ROOT
for h in "" 3000 12000 25000; do
FP_L2B_HOT=$h timeout 600 python bench.py --config K1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K1 hot=$h', d['ms_per_step'], d['roofline']['frac'], d['config']['packed_copy']['detail']['hot_columns'])"
done

#!/bin/bash
cd $GRAFT_REPO_ROOT
for mg in 0 1; do for h in 6000 20000 60000; do
FP_L2B_MERGE=$mg FP_L2B_HOT=$h timeout 600 python bench.py --config K1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K1 merge=$mg hot=$h', d['ms_per_step'], d['roofline']['frac'], d['gpu_launches'])"
done; done

#!/bin/bash
cd $GRAFT_REPO_ROOT
for c in C3 S3; do
for bs in 512 768 1024; do
FP_PK_BS1=$bs timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$c bs=$bs ms', d['ms_per_step'], d['roofline']['frac'], d['config']['plan']['variant'])"
done; done

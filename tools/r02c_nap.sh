#!/bin/bash
cd $GRAFT_REPO_ROOT
for r in 1 2 3; do for nap in 0 -100; do
FP_PK_NAP=$nap timeout 600 python bench.py --config C4 --steps 20 --warmup 5 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4 nap=$nap', d['ms_per_step'], d['roofline']['frac'])"
done; done

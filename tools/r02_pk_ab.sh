#!/bin/bash
cd $GRAFT_REPO_ROOT
for pf in 1 0 2; do
FP_PK_PF=$pf timeout 300 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('pf=$pf ms', d['ms_per_step'], d['roofline']['frac'])"
done

#!/bin/bash
cd $GRAFT_REPO_ROOT
for rt in "4 0" "4 128" "4 512" "0 256" "12 0" "4 0"; do
set -- $rt
FP_PK_ROWCOST=$1 FP_PK_TILECOST=$2 timeout 600 python bench.py --config C4 --steps 20 --warmup 5 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4 rc=$1 tc=$2', d['ms_per_step'], d['roofline']['frac'])"
done

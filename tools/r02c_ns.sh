#!/bin/bash
cd $GRAFT_REPO_ROOT
for r in 1 2; do for ns in 2 3 4; do
FP_PK1_NS=$ns timeout 600 python bench.py --config C3 --steps 20 --warmup 5 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C3 ns=$ns', d['ms_per_step'], d['roofline']['frac'])"
done; done

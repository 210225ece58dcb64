#!/bin/bash
cd $GRAFT_REPO_ROOT
for L in "1,32,4,32" "1,32,4,64" "1,32,4,125" "1,32,4,250" "1,16,8,64" "1,16,8,125" "1,8,16,125" "1,4,32,250"; do
timeout 300 python bench.py --config C1 --steps 200 --warmup 20 --no-e2e --no-cpu-baseline --launch $L 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C1 $L', d['ms_per_step']*1000, 'us', d['config']['plan'])" 2>&1 | tail -1
done

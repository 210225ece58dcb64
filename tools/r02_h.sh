#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_binned_gpu.py -x -q 2>&1 | tail -2
for v in 19 7 16; do
timeout 600 python bench.py --config K1 --launch $v,32,8,0 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K1 v$v', d['ms_per_step'])"
done
timeout 600 python bench.py --config C4 --launch 19,32,8,0 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4 v19', d['ms_per_step'])"

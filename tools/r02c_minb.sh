#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x -k "l2block" 2>&1 | tail -1
for i in 1 2 3; do
timeout 600 python bench.py --config K1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K1', d['ms_per_step'], d['roofline']['frac'])"
done

#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x -k "packed1 or detail" 2>&1 | tail -1
for r in 1 2; do for c in C3 S3; do
timeout 600 python bench.py --config $c --steps 20 --warmup 5 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', d['ms_per_step'], d['roofline']['frac'])"
done; done

#!/bin/bash
cd $GRAFT_REPO_ROOT
for i in 1 2 3; do
timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x -k "packed1 or pack_detail" 2>&1 | tail -1
done
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -p no:cacheprovider --timeout 600 -rf -k "packed and C3" 2>&1 | tail -1
for i in 1 2; do
timeout 600 python bench.py --config C3 --steps 20 --warmup 5 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C3', d['ms_per_step'], d['roofline']['frac'])"
done

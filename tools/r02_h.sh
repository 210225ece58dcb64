#!/bin/bash
cd $GRAFT_REPO_ROOT
FP_BIN_NT4=1 timeout 900 python -m pytest tests/test_binned_gpu.py -x -q -k binned 2>&1 | tail -2
for e in 1 0 1 0; do
FP_BIN_NT4=$e timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4 nt4=$e', d['ms_per_step'])"
done

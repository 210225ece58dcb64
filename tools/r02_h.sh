#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
FP_BIN_EMIT=1 timeout 900 python -m pytest tests/test_binned_gpu.py -x -q -k "binned" 2>&1 | tail -3
for e in 0 1 0 1; do
FP_BIN_EMIT=$e timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('emit', $e, d['ms_per_step'])"
done

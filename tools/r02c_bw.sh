#!/bin/bash
cd $GRAFT_REPO_ROOT
for bw in 4194304 6291456 8388608 12582912; do
FP_L2B_BW=$bw timeout 600 python bench.py --config K1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K1 bw=$bw', d['ms_per_step'], d['roofline']['frac'], d['config']['packed_copy']['blocks'])"
done

#!/bin/bash
# variant 20: packed tests, K1 bench over block widths
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x 2>&1 | tail -4
for bw in 1048576 2097152 4194304; do
FP_L2B_BW=$bw timeout 600 python bench.py --config K1 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>gpurun_out/k1_$bw.err | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('K1 bw=$bw ms', d['ms_per_step'], d['roofline']['frac'], d['config'].get('plan',{}).get('variant'), d['config'].get('packed_copy'))" 2>&1 | tail -2
done

#!/bin/bash
# A/B of the wide-row dense cluster kernels (register-only vs bulk-copy ring; slice width;
# ring depth) on config ${W:-W1}: prints ms/step, roofline fraction, chosen plan.
mkdir -p gpurun_out
for cfg in "0 256 3" "0 128 3" "1 128 3" "1 128 2" "1 128 4"; do
  set -- $cfg
  FP_CLUSTER_TMA=$1 FP_CLUSTER_TB=$2 FP_CLUSTER_RING=$3 python bench.py --config ${W:-W1} --steps 10 --warmup 3 2>/dev/null | tail -1 \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('tma=$1 tb=$2 ring=$3', d['ms_per_step'], d['roofline']['frac'], d['config'].get('plan'), d['clocks']['reasons'])"
done

#!/bin/bash
cd $GRAFT_REPO_ROOT
for h in 1500 3000 4500; do
FP_L2B_HOT=$h timeout 600 python bench.py --config K1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K1 hot=$h', d['ms_per_step'], d['roofline']['frac'])"
done
bash tools/ncu_one.sh '^k_pk1$' C3 r02c_C3b
python tools/ncu_stalls.py gpurun_out/r02c_C3b_source.csv 30 > gpurun_out/r02c_C3b_stalls.txt
head -3 gpurun_out/r02c_C3b_stalls.txt

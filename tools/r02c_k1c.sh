#!/bin/bash
cd $GRAFT_REPO_ROOT
for h in "" 0 20000; do
FP_L2B_HOT=$h timeout 600 python bench.py --config K1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K1 hot=$h', d['ms_per_step'], d['roofline']['frac'], d['config'].get('packed_copy'))"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02c_K1_launches.csv python bench.py --config K1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/r02c_K1_launches.csv 2>&1 | grep "k_l2b" | grep -v "walk\|count\|scatter\|fill\|rows\|hotsel\|gather\|blocktot\|hotrows"

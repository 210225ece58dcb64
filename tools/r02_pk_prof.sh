#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/pk_c4.json 2> gpurun_out/pk_c4.err
python -c "
import json; d=json.loads(open('gpurun_out/pk_c4.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['roofline']['frac'])"
timeout 900 ncu --set full --clock-control none --import-source on -k k_pk -c 1 -o gpurun_out/pk_c4_full -f python bench.py --config C4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > gpurun_out/pk_ncu.log 2>&1
tail -1 gpurun_out/pk_ncu.log

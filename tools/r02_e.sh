#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_binned_gpu.py -x -q 2>&1 | tail -25 > gpurun_out/r02e_tests.txt
for v in 19 18 3; do for c in C3 S3; do
timeout 600 python bench.py --config $c --launch $v,4,4,0 --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02e_${c}_v$v.json 2>> gpurun_out/r02e_c3.err
done; done
cat gpurun_out/r02e_tests.txt; for f in gpurun_out/r02e_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', d['ms_per_step'], d['roofline']['frac'])"; done; tail -3 gpurun_out/r02e_c3.err

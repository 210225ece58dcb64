#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for pf in 256 512 1024 2048; do
FP_BIN_PF=$pf timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02f_c4_pf$pf.json 2>> gpurun_out/r02f.err
FP_BIN_PF=$pf timeout 600 python bench.py --config C3 --launch 18,4,4,0 --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02f_c3_pf$pf.json 2>> gpurun_out/r02f.err
done
for f in gpurun_out/r02f_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', d['ms_per_step'], d['roofline']['frac'])"; done; tail -3 gpurun_out/r02f.err

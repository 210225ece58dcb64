#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python tools/sweep.py --config C3 --reps 5 --out gpurun_out/r02_sweep_C3.json > gpurun_out/r02_sweep_C3.log 2>&1
timeout 1200 python tools/sweep.py --config S3 --reps 5 --out gpurun_out/r02_sweep_S3.json > gpurun_out/r02_sweep_S3.log 2>&1
timeout 1800 python tools/sweep.py --config C4 --reps 3 --variants 4,7,16,17 --out gpurun_out/r02_sweep_C4.json > gpurun_out/r02_sweep_C4.log 2>&1
tail -2 gpurun_out/r02_sweep_*.log

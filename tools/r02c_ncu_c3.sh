#!/bin/bash
# source-level stall capture of the single-block packed pass (C3 fp64, S3 fp32)
cd $GRAFT_REPO_ROOT
for c in C3 S3; do
bash tools/ncu_one.sh '^k_pk1$' $c r02c_${c}
python tools/ncu_stalls.py gpurun_out/r02c_${c}_source.csv 40 > gpurun_out/r02c_${c}_stalls.txt
head -45 gpurun_out/r02c_${c}_stalls.txt
done

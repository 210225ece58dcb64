#!/bin/bash
cd $GRAFT_REPO_ROOT
bash tools/ncu_one.sh '^k_pk1$' C3 r02c_C3c
python tools/ncu_stalls.py gpurun_out/r02c_C3c_source.csv 40 > gpurun_out/r02c_C3c_stalls.txt
head -42 gpurun_out/r02c_C3c_stalls.txt

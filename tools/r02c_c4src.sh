#!/bin/bash
cd $GRAFT_REPO_ROOT
bash tools/ncu_one.sh '^k_pk$' C4 r02c_C4s
python tools/ncu_stalls.py gpurun_out/r02c_C4s_source.csv 40 > gpurun_out/r02c_C4s_stalls.txt
head -45 gpurun_out/r02c_C4s_stalls.txt

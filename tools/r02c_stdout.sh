#!/bin/bash
cd $GRAFT_REPO_ROOT
NCCL_DEBUG=WARN timeout 600 python bench.py --config C2 --force-dist --exchange nccl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null > gpurun_out/stdout_check.txt
wc -l gpurun_out/stdout_check.txt; cut -c1-120 gpurun_out/stdout_check.txt
timeout 600 python bench.py --config C1 --steps 5 --warmup 3 2>/dev/null | wc -l

#!/bin/bash
# round-2 GPU check: binned variant parity + C4 bench A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_binned_gpu.py tests/test_dist_nccl_gpu.py -x -q 2>&1 | tail -30 > gpurun_out/r02a_tests.txt
timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02a_c4.json 2> gpurun_out/r02a_c4.err
FP_NO_BINNED=1 timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02a_c4_v16.json 2>> gpurun_out/r02a_c4.err
timeout 1200 python -m pytest tests/test_parity_csr_gpu.py tests/test_parity_dense_gpu.py -x -q 2>&1 | tail -15 > gpurun_out/r02a_tests2.txt
cat gpurun_out/r02a_tests.txt; cat gpurun_out/r02a_c4.json gpurun_out/r02a_c4_v16.json; tail -5 gpurun_out/r02a_c4.err; cat gpurun_out/r02a_tests2.txt

set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_csr_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -3
bash tools/plan_bench.sh C4 7,32,8,0 7,32,4,0 7,32,2,0
bash tools/plan_bench.sh C3 3,8,2,0 3,2,4,0 11,4,4,0 11,8,2,0 12,32,4,0 12,32,2,0

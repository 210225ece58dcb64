set -u
FP_L2_REPLICAS=3 timeout 900 python -m pytest tests/test_parity_csr_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -2
for r in 1 2 4 8 16; do echo "rep=$r"; FP_L2_REPLICAS=$r bash tools/plan_bench.sh C4 7,32,8,0; done
FP_L2_REPLICAS=8 bash tools/plan_bench.sh C4 4,32,4,0 7,32,4,0

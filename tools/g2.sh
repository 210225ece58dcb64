set -u
mkdir -p gpurun_out
bash tools/plan_bench.sh C3 3,8,2,0 3,2,4,0 11,8,2,0 11,2,4,0 11,4,4,0 11,2,8,0 12,32,2,0 12,32,4,0 12,32,8,0 6,32,4,0 > gpurun_out/plans_C3.txt 2>&1
bash tools/plan_bench.sh C4 7,32,8,0 7,32,4,0 13,32,8,4 > gpurun_out/plans_C4.txt 2>&1
cat gpurun_out/plans_C3.txt gpurun_out/plans_C4.txt

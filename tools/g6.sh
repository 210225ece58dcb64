set -u
mkdir -p gpurun_out
timeout 900 python tools/sweep.py --config C3 --variants 3,11,12 --grids 296,592,888 --out gpurun_out/sweep_C3.json 2>&1 | tail -2
timeout 900 python tools/sweep.py --config S3 --variants 3,11,12 --grids 296,592,888 --out gpurun_out/sweep_S3.json 2>&1 | tail -2
bash tools/plan_bench.sh C4 7,32,8,0

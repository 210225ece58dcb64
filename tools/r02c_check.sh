#!/bin/bash
# round-2c re-entry check: GPU suite, smoke, C4 / C3 / S3 bench lines on HEAD
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 600 python bench.py > gpurun_out/r02c_C4.json 2> gpurun_out/r02c_C4.err; tail -c 600 gpurun_out/r02c_C4.json
for c in C3 S3; do
timeout 600 python bench.py --config $c --steps 20 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/r02c_$c.json 2>> gpurun_out/r02c_C4.err
python -c "import json; d=json.load(open('gpurun_out/r02c_$c.json')); print('$c', d['ms_per_step'], d['roofline']['frac'], d['config']['plan'].get('variant'))"
done
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 -rf -x > gpurun_out/r02c_pytest_gpu.log 2>&1
tail -3 gpurun_out/r02c_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1

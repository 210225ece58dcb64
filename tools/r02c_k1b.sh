#!/bin/bash
# variant 20 after the pack fixes: tests, full-size packed parity, K1 bench, ncu of the passes
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x -k l2block 2>&1 | tail -3
timeout 1500 python -m pytest tests/test_fullsize_gpu.py -q -p no:cacheprovider --timeout 900 -rf -k packed 2>&1 | tail -4
timeout 600 python bench.py --config K1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>gpurun_out/k1.err | tail -1 > gpurun_out/r02c_K1.json
python -c "import json; d=json.load(open('gpurun_out/r02c_K1.json')); print('K1', d['ms_per_step'], d['roofline']['frac'], d['config'].get('packed_copy'), d['roofline'].get('second_ceiling',{}).get('floor_ms'))"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_l2b$ --launch-skip 0 --launch-count 16 -o gpurun_out/r02c_K1_full -f python bench.py --config K1 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c_K1_full.ncu-rep --page raw --csv > gpurun_out/r02c_K1_raw.csv 2>/dev/null
ncu -i gpurun_out/r02c_K1_full.ncu-rep --page details --csv > gpurun_out/r02c_K1_details.csv 2>/dev/null
rm -f gpurun_out/r02c_K1_full.ncu-rep

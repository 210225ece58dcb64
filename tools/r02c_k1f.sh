#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py tests/test_fullsize_gpu.py -q -p no:cacheprovider --timeout 900 -rf -k "l2block or detail or K1" 2>&1 | tail -1
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python bench.py --config K1 --steps 20 --warmup 5 > gpurun_out/r02c4_K1.json 2>/dev/null; python -c "import json; d=json.loads(open('gpurun_out/r02c4_K1.json').read().strip().splitlines()[-1]); print('K1', d['ms_per_step'], d['roofline']['frac'], d['gpu_launches'], d['config']['packed_copy'])"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02c4_K1_launches.csv python bench.py --config K1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none -k regex:"^k_l2b(_init|_q|_hot)?$" -c 19 -o gpurun_out/r02c4_K1_full -f python bench.py --config K1 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c4_K1_full.ncu-rep --page raw --csv > gpurun_out/r02c4_K1_raw.csv 2>/dev/null
rm -f gpurun_out/r02c4_K1_full.ncu-rep

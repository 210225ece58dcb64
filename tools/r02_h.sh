#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_binned_gpu.py -x -q -k "binned" 2>&1 | tail -2
for i in 1 2; do
timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4', d['ms_per_step'])"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:k_bin" --csv --log-file gpurun_out/r02h_launches.csv python bench.py --config C4 --steps 1 --warmup 3 --no-graph --no-e2e --no-cpu-baseline > /dev/null 2>&1
grep -v "^==" gpurun_out/r02h_launches.csv | cut -d, -f5,15- | tail -3

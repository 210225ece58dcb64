#!/bin/bash
# round-2 re-check after variant 19: full GPU suite, smoke, default bench line, C4 launch list +
# ncu --set full captures of the packed pass and its finalize
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 -rf > gpurun_out/pytest_gpu.log 2>&1
tail -4 gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r02b_bench_C4.json 2> gpurun_out/r02b_bench_C4.err
python -c "
import json; d=json.loads(open('gpurun_out/r02b_bench_C4.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['value'], d['roofline']['frac'], (d.get('e2e') or {}).get('value'), (d.get('cpu_baseline') or {}).get('value'))"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02b_C4_launches.csv python bench.py --config C4 --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_pk(_finalize)?$" -c 2 -o gpurun_out/r02b_C4_full -f python bench.py --config C4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > gpurun_out/r02b_ncu.log 2>&1
ncu -i gpurun_out/r02b_C4_full.ncu-rep --page raw --csv > gpurun_out/r02b_C4_raw.csv 2>/dev/null
tail -2 gpurun_out/r02b_ncu.log

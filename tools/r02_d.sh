#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for c in C4 C3; do
timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02d_$c.json 2> gpurun_out/r02d_$c.err
done
timeout 900 python bench.py --config C4 --cols iid --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02d_C4iid.json 2> gpurun_out/r02d_C4iid.err
for f in gpurun_out/r02d_*.json; do python -c "
import json,sys; d=json.load(open('$f')); r=d['roofline']; print('$f', d['ms_per_step'], r['frac'], r['binding'], json.dumps(r['second_ceiling']), r['traffic_source'])"; done
tail -2 gpurun_out/r02d_*.err

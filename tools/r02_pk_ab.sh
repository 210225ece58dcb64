#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_peer_exchange_gpu.py tests/test_drivers_gpu.py tests/test_dist_nccl_gpu.py -q -x -p no:cacheprovider --timeout 300 2>&1 | tail -3
for ex in peer nccl; do
timeout 300 python bench.py --config C4 --force-dist --exchange $ex --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('dist $ex ms', d['ms_per_step'], d['roofline']['frac'], d['config']['parallelism'])"
done

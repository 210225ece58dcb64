#!/bin/bash
cd $GRAFT_REPO_ROOT
FP_PK_BSN=768 timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x -k "packed_ and not packed1" 2>&1 | tail -2
for bsn in 1024 768; do
FP_PK_BSN=$bsn timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4 bsn=$bsn', d['ms_per_step'], d['roofline']['frac'])"
done

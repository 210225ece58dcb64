#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x 2>&1 | tail -2
for c in C4 C3 S3; do for ls in 0 1; do
if [ $ls = 0 ]; then export FP_PK_NOLS=1; else unset FP_PK_NOLS; fi
timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c ls=$ls', d['ms_per_step'], d['roofline']['frac'], d['config']['packed_copy']['pack_ms'])"
done; done

#!/bin/bash
cd $GRAFT_REPO_ROOT
FP_PK_BS1=640 timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x -k "packed1" 2>&1 | tail -2
for c in C3 S3; do for bs in 512 640 768 1024; do
FP_PK_BS1=$bs timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c bs=$bs', d['ms_per_step'], d['roofline']['frac'])"
done; done

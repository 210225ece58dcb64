#!/bin/bash
# variant 19 A/B: L2 hints and poll sleep
cd $GRAFT_REPO_ROOT
for pol in 1,2 0,0 0,2 1,0; do for nap in 64 0; do
  echo "== FP_PK_POL=$pol FP_PK_NAP=$nap"
  FP_PK_POL=$pol FP_PK_NAP=$nap timeout 300 python tools/pk_trace.py C4 2>/dev/null | grep -E "end us perc|poll wait|dot ms"
  FP_PK_POL=$pol FP_PK_NAP=$nap timeout 300 python bench.py --config C4 --steps 5 --warmup 2 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('ms', d['ms_per_step'])"
done; done

#!/bin/bash
# Time explicit CSR plans through bench.py (grid 0 = one resident wave):
#   tools/plan_bench.sh C3 11,2,4,0 3,8,2,0 ...
cfg=$1; shift
for P in "$@"; do
  echo -n "$cfg $P "
  timeout 300 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --launch $P |
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['kernel_ms'], 'ms  frac', d['roofline']['frac'])"
done

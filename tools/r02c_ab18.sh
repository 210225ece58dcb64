#!/bin/bash
# A/B of variant 18's grouped limb atomics (C3 through the unpacked chooser plan): the in-tree
# library (grouped), then the FP_FIX_NOGROUP build copied over it (on the box's copy only)
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_binned_gpu.py tests/test_parity_csr_gpu.py -q -p no:cacheprovider --timeout 300 -x -k "flat4 or fixed_point" 2>&1 | tail -1
for v in group nogroup; do
  if [ $v = nogroup ]; then cp gpurun_ab/libfusedpat_nogroup.so paper_conf_ppopp_asharitbrcks15_b200/libfusedpat.so; fi
  for i in 1 2; do
  timeout 600 python bench.py --config C3 --no-pack --steps 20 --warmup 5 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C3 unpacked $v', d['ms_per_step'], d['roofline']['frac'], d['config']['plan']['variant'])"
  done
done

#!/bin/bash
# binned variant: parity + C4 bench + launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_binned_gpu.py tests/test_drivers_gpu.py tests/test_logreg_gpu.py -x -q 2>&1 | tail -30 > gpurun_out/r02b_tests.txt
timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02b_c4.json 2> gpurun_out/r02b_c4.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:k_bin" --csv \
  --log-file gpurun_out/r02b_launches.csv python bench.py --config C4 --steps 2 --warmup 3 --no-graph --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_bin_produce" -s 1 -c 1 \
  -o gpurun_out/r02b_prod -f python bench.py --config C4 --steps 1 --warmup 3 --no-graph --no-e2e --no-cpu-baseline > /dev/null 2>&1
cat gpurun_out/r02b_tests.txt; cat gpurun_out/r02b_c4.json; tail -3 gpurun_out/r02b_c4.err; grep -v "^==" gpurun_out/r02b_launches.csv | cut -d, -f5,15- | tail -6

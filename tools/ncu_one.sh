#!/bin/bash
# ncu --set full of the first launch of kernel regex $1 under `python bench.py --config $2`;
# exports raw/source/details CSVs as gpurun_out/$3_*.csv and drops the .ncu-rep (size cap).
set -u
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k "regex:$1" -c 1 -o "gpurun_out/$3" \
  python bench.py --config "$2" --steps 1 --warmup 3 > "gpurun_out/$3_bench.log" 2>&1
for p in raw details; do ncu -i "gpurun_out/$3.ncu-rep" --page $p --csv > "gpurun_out/$3_$p.csv"; done
ncu -i "gpurun_out/$3.ncu-rep" --page source --csv --print-source sass > "gpurun_out/$3_source.csv"
rm -f "gpurun_out/$3.ncu-rep"

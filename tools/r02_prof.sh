#!/bin/bash
# usage: tools/r02_prof.sh TAG CONFIG KREGEX [extra bench args]  -- launch list + one full capture
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=$1; CFG=$2; KRE=$3; shift 3
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:$KRE" --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --config $CFG --steps 2 --warmup 3 --no-graph --no-e2e --no-cpu-baseline "$@" > gpurun_out/${TAG}_launches.log 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k "regex:$KRE" -s 3 -c 3 \
  -o gpurun_out/${TAG}_full -f python bench.py --config $CFG --steps 1 --warmup 3 --no-graph --no-e2e --no-cpu-baseline "$@" > gpurun_out/${TAG}_full.log 2>&1
grep -v "^==" gpurun_out/${TAG}_launches.csv | tail -20

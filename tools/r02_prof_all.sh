#!/bin/bash
# round-2 evidence: launch list + one ncu --set full capture per config (1 GPU)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
KRE="k_dense_|k_csr_vector|k_csr_flat|k_flat4|k_bin_|k_cg_|k_scale_z|k_fold"
run() {  # tag config full-regex skip count extra-args
  local TAG=$1 CFG=$2 FRE=$3 SKIP=$4 CNT=$5; shift 5
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:$KRE" --csv \
    --log-file gpurun_out/${TAG}_launches.csv python bench.py --config $CFG --steps 2 --warmup 3 --no-graph --no-e2e --no-cpu-baseline "$@" > gpurun_out/${TAG}_launches.log 2>&1
  timeout 1500 ncu --set full --clock-control none --import-source on -k "regex:$FRE" -s $SKIP -c $CNT \
    -o /tmp/${TAG}_full -f python bench.py --config $CFG --steps 1 --warmup 3 --no-graph --no-e2e --no-cpu-baseline "$@" > gpurun_out/${TAG}_full.log 2>&1
  ncu -i /tmp/${TAG}_full.ncu-rep --page raw --csv > gpurun_out/${TAG}_raw.csv 2>/dev/null
  ncu -i /tmp/${TAG}_full.ncu-rep --page details --csv > gpurun_out/${TAG}_details.csv 2>/dev/null
  ncu -i /tmp/${TAG}_full.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/${TAG}_source.csv 2>/dev/null
  gzip -f gpurun_out/${TAG}_source.csv
  echo "$TAG done $(ls -la /tmp/${TAG}_full.ncu-rep 2>/dev/null | awk '{print $5}')"
}
run r02_C4 C4 "k_flat4|k_bin_" 9 3
run r02_C3 C3 "k_flat4" 3 1
run r02_C2 C2 "k_dense_vector" 3 1
run r02_C1 C1 "k_dense_vector" 3 1
run r02_C5 C5 "k_dense_vector" 5 1 --cg-iters 2

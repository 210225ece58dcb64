#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
KRE="k_csr_flat|k_scale_z|k_fold"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:$KRE" --csv \
    --log-file gpurun_out/r02_K1_launches.csv python bench.py --config K1 --steps 2 --warmup 3 --no-graph --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k "regex:k_csr_flat" -s 3 -c 1 \
    -o /tmp/r02_K1_full -f python bench.py --config K1 --steps 1 --warmup 3 --no-graph --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/r02_K1_full.ncu-rep --page raw --csv > gpurun_out/r02_K1_raw.csv 2>/dev/null
ncu -i /tmp/r02_K1_full.ncu-rep --page details --csv > gpurun_out/r02_K1_details.csv 2>/dev/null
ncu -i /tmp/r02_K1_full.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/r02_K1_source.csv 2>/dev/null; gzip -f gpurun_out/r02_K1_source.csv
echo done

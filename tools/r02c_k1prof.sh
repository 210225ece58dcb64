#!/bin/bash
# K1 on variant 20: launch list of one step, full capture of a dot, the fused and a scatter pass
cd $GRAFT_REPO_ROOT
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/r02c_K1_launches.csv python bench.py --config K1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/r02c_K1_launches.csv 2>&1 | tail -60
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_l2b --launch-skip 0 --launch-count 16 -o gpurun_out/r02c_K1_full -f python bench.py --config K1 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c_K1_full.ncu-rep --page raw --csv > gpurun_out/r02c_K1_raw.csv 2>/dev/null
ncu -i gpurun_out/r02c_K1_full.ncu-rep --page details --csv > gpurun_out/r02c_K1_details.csv 2>/dev/null
rm -f gpurun_out/r02c_K1_full.ncu-rep

#!/bin/bash
# variant 20: packed tests, K1 bench over block widths
cd $GRAFT_REPO_ROOT
: timeout 900 python -m pytest tests/test_packed_gpu.py -q -p no:cacheprovider --timeout 300 -rf -x 2>&1 | tail -4
for bw in 4194304 8388608 16777216; do
FP_L2B_BW=$bw timeout 600 python bench.py --config K1 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>gpurun_out/k1_$bw.err | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('K1 bw=$bw ms', d['ms_per_step'], d['roofline']['frac'], d['config'].get('plan',{}).get('variant'), d['config'].get('packed_copy'))" 2>&1 | tail -2
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/r02c_K1_launches.csv python bench.py --config K1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/r02c_K1_launches.csv 2>&1 | grep -v "k_probe\|cub::\|k_csr_fill\|k_vector\|k_row_len\|k_csr_check" | head -30

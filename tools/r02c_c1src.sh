#!/bin/bash
cd $GRAFT_REPO_ROOT
bash tools/ncu_one.sh 'k_dense_vector' C1 r02c_C1s
python tools/ncu_stalls.py gpurun_out/r02c_C1s_source.csv 25 | head -28
python - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/r02c_C1s_raw.csv')))
h=rows[0]
for k in ['gpu__time_duration.sum','smsp__inst_executed.sum','launch__grid_size','launch__block_size','sm__warps_active.avg.pct_of_peak_sustained_active','dram__bytes_read.sum']:
    if k in h: print(k, rows[2][h.index(k)])
PY

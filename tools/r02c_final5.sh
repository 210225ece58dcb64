#!/bin/bash
# last HEAD check: GPU suite, smoke, bench lines (default C4, C3, S3, K1), C3 captures
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 -rf > gpurun_out/r02c7_pytest_gpu.log 2>&1
tail -2 gpurun_out/r02c7_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
OUT=gpurun_out/r02c7_bench.jsonl
: > $OUT
timeout 900 python bench.py >> $OUT 2> gpurun_out/r02c7.err
for c in C3 S3 K1; do timeout 900 python bench.py --config $c --steps 20 --warmup 5 >> $OUT 2>> gpurun_out/r02c7.err; done
python - <<'PY'
import json
for ln in open("gpurun_out/r02c7_bench.jsonl"):
    d = json.loads(ln)
    r = d.get("roofline") or {}
    print(d["config"]["workload"][:30], d.get("ms_per_step"), d.get("value"), r.get("frac"), (d.get("e2e") or {}).get("value"), (d.get("cpu_baseline") or {}).get("value"), d.get("gpu_launches"), d.get("clocks", {}).get("reasons"))
PY
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02c7_C3_launches.csv python bench.py --config C3 --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_pk1(_finalize)?$" -c 2 -o gpurun_out/r02c7_C3_full -f python bench.py --config C3 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c7_C3_full.ncu-rep --page raw --csv > gpurun_out/r02c7_C3_raw.csv 2>/dev/null
rm -f gpurun_out/r02c7_C3_full.ncu-rep

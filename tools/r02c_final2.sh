#!/bin/bash
# round-2c final re-check after the C3 / C4 changes: GPU suite, smoke, bench lines, C3/C4 captures
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 -rf > gpurun_out/r02c2_pytest_gpu.log 2>&1
tail -2 gpurun_out/r02c2_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
OUT=gpurun_out/r02c2_final_bench.jsonl
: > $OUT
timeout 900 python bench.py >> $OUT 2> gpurun_out/r02c2_final.err
for c in C1 C2 C3 C5 S3 W1 K1; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 5 >> $OUT 2>> gpurun_out/r02c2_final.err
done
timeout 900 python bench.py --config C4 --impl reference >> $OUT 2>> gpurun_out/r02c2_final.err
python - <<'PY'
import json
for ln in open("gpurun_out/r02c2_final_bench.jsonl"):
    try:
        d = json.loads(ln)
    except Exception:
        continue
    r = d.get("roofline") or {}
    pl = (d.get("config") or {}).get("plan") or {}
    print(d.get("impl", "fusedpat"), d["config"]["workload"][:30], pl.get("variant"), d.get("ms_per_step"), d.get("value"), r.get("frac"),
          (d.get("e2e") or {}).get("value"), (d.get("cpu_baseline") or {}).get("value"), d.get("gpu_launches"), (r.get("second_ceiling") or {}).get("frac"), d.get("clocks", {}).get("reasons"))
PY
for c in C3 C4; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02c2_${c}_launches.csv python bench.py --config $c --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_pk1(_finalize)?$" -c 2 -o gpurun_out/r02c2_C3_full -f python bench.py --config C3 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c2_C3_full.ncu-rep --page raw --csv > gpurun_out/r02c2_C3_raw.csv 2>/dev/null
rm -f gpurun_out/r02c2_C3_full.ncu-rep
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_pk(_finalize)?$" -c 2 -o gpurun_out/r02c2_C4_full -f python bench.py --config C4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c2_C4_full.ncu-rep --page raw --csv > gpurun_out/r02c2_C4_raw.csv 2>/dev/null
rm -f gpurun_out/r02c2_C4_full.ncu-rep

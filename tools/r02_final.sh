#!/bin/bash
# round-2 measurements: every config through bench.py (CUDA events, graphs), the reference and
# unfused arms for C4, the 1-rank dist paths, the C3 sweep with the final chooser
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
OUT=gpurun_out/r02_final_bench.jsonl
: > $OUT
timeout 900 python bench.py >> $OUT 2> gpurun_out/r02_final.err          # the default line (C4)
for c in C1 C2 C3 C5 S3 W1 K1; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 5 >> $OUT 2>> gpurun_out/r02_final.err
done
timeout 900 python bench.py --config C4 --cols iid --no-e2e --no-cpu-baseline >> $OUT 2>> gpurun_out/r02_final.err
FP_NO_BINNED=1 timeout 900 python bench.py --config C4 --no-e2e --no-cpu-baseline >> $OUT 2>> gpurun_out/r02_final.err
for ex in peer nccl; do
  timeout 900 python bench.py --config C4 --force-dist --exchange $ex --no-e2e --no-cpu-baseline >> $OUT 2>> gpurun_out/r02_final.err
done
timeout 900 python bench.py --config C4 --impl reference >> $OUT 2>> gpurun_out/r02_final.err
timeout 900 python bench.py --config C4 --impl unfused --steps 3 --warmup 3 >> $OUT 2>> gpurun_out/r02_final.err
timeout 1500 python tools/sweep.py --config C3 --reps 5 --out gpurun_out/r02_sweep_C3.json > gpurun_out/r02_sweep_C3.log 2>&1
python - <<'PY'
import json
for ln in open("gpurun_out/r02_final_bench.jsonl"):
    try:
        d = json.loads(ln)
    except Exception:
        continue
    r = d.get("roofline") or {}
    print(d.get("impl", "fusedpat"), d["config"]["workload"][:40], d.get("ms_per_step"), d.get("value"), r.get("frac"),
          r.get("binding"), (d.get("e2e") or {}).get("value"), (d.get("cpu_baseline") or {}).get("value"),
          d["config"].get("parallelism"))
PY
tail -n 3 gpurun_out/r02_sweep_C3.log | cut -c1-600
tail -n 5 gpurun_out/r02_final.err

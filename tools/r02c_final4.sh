#!/bin/bash
# HEAD re-check at the end of round 2c: GPU suite, smoke, every config's bench line
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 -rf > gpurun_out/r02c5_pytest_gpu.log 2>&1
tail -2 gpurun_out/r02c5_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
OUT=gpurun_out/r02c5_final_bench.jsonl
: > $OUT
timeout 900 python bench.py >> $OUT 2> gpurun_out/r02c5.err
for c in C1 C2 C3 C5 S3 W1 K1; do timeout 900 python bench.py --config $c --steps 20 --warmup 5 >> $OUT 2>> gpurun_out/r02c5.err; done
timeout 900 python bench.py --impl reference >> $OUT 2>> gpurun_out/r02c5.err
timeout 900 python bench.py --config C4 --force-dist --exchange peer --no-e2e --no-cpu-baseline >> $OUT 2>> gpurun_out/r02c5.err
python - <<'PY'
import json
for ln in open("gpurun_out/r02c5_final_bench.jsonl"):
    try:
        d = json.loads(ln)
    except Exception:
        print("NONJSON", ln[:80]); continue
    r = d.get("roofline") or {}
    print(d.get("impl", "fusedpat"), d["config"]["workload"][:30], d.get("ms_per_step"), d.get("value"), r.get("frac"), (d.get("e2e") or {}).get("value"), (d.get("cpu_baseline") or {}).get("value"), d.get("gpu_launches"), d.get("clocks", {}).get("reasons"), d["config"].get("parallelism"))
PY

#!/bin/bash
# round-2c measurements: full GPU suite, smoke, every config through bench.py, C4 arms,
# launch lists + ncu --set full of the dominant kernels (C4, C3, S3, K1)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 -rf > gpurun_out/r02c_pytest_gpu.log 2>&1
tail -3 gpurun_out/r02c_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
OUT=gpurun_out/r02c_final_bench.jsonl
: > $OUT
timeout 900 python bench.py >> $OUT 2> gpurun_out/r02c_final.err
for c in C1 C2 C3 C5 S3 W1 K1; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 5 >> $OUT 2>> gpurun_out/r02c_final.err
done
timeout 900 python bench.py --config C4 --cols iid --no-e2e --no-cpu-baseline >> $OUT 2>> gpurun_out/r02c_final.err
timeout 900 python bench.py --config K1 --no-pack --no-e2e --no-cpu-baseline --steps 5 --warmup 3 >> $OUT 2>> gpurun_out/r02c_final.err
for ex in peer nccl; do
  timeout 900 python bench.py --config C4 --force-dist --exchange $ex --no-e2e --no-cpu-baseline >> $OUT 2>> gpurun_out/r02c_final.err
done
timeout 900 python bench.py --config C4 --impl reference >> $OUT 2>> gpurun_out/r02c_final.err
python - <<'PY'
import json
for ln in open("gpurun_out/r02c_final_bench.jsonl"):
    try:
        d = json.loads(ln)
    except Exception:
        continue
    r = d.get("roofline") or {}
    pl = (d.get("config") or {}).get("plan") or {}
    print(d.get("impl", "fusedpat"), d["config"]["workload"][:30], pl.get("variant"), d.get("ms_per_step"), d.get("value"), r.get("frac"),
          (d.get("e2e") or {}).get("value"), (d.get("cpu_baseline") or {}).get("value"), d["config"].get("parallelism"), d.get("gpu_launches"))
PY
for c in C3 S3 C4 K1; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02c_${c}_launches.csv python bench.py --config $c --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
done
for c in C3 S3; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_pk1(_finalize)?$" -c 2 -o gpurun_out/r02c_${c}_full -f python bench.py --config $c --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c_${c}_full.ncu-rep --page raw --csv > gpurun_out/r02c_${c}_raw.csv 2>/dev/null
rm -f gpurun_out/r02c_${c}_full.ncu-rep
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_pk(_finalize)?$" -c 2 -o gpurun_out/r02c_C4_full -f python bench.py --config C4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c_C4_full.ncu-rep --page raw --csv > gpurun_out/r02c_C4_raw.csv 2>/dev/null
rm -f gpurun_out/r02c_C4_full.ncu-rep
timeout 1200 ncu --set full --clock-control none -k regex:"^k_l2b(_init|_q|_hot)?$" -c 33 -o gpurun_out/r02c_K1_full -f python bench.py --config K1 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
ncu -i gpurun_out/r02c_K1_full.ncu-rep --page raw --csv > gpurun_out/r02c_K1_raw.csv 2>/dev/null
rm -f gpurun_out/r02c_K1_full.ncu-rep
ls -la gpurun_out | head -50

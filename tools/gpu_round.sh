#!/bin/bash
# One GPU session: tests, benches, ncu evidence.  Outputs under gpurun_out/.
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 -rf > gpurun_out/pytest_gpu.log 2>&1
tail -3 gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -c 300 gpurun_out/bench_default.json
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in C1 C3 C4 C5 S3 W1 K1; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
# launch list of the default bench command (and of C3 / C4)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_C2.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
for c in C3 C4; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$c.csv python bench.py --config $c --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
KR="regex:k_dense_vector|k_csr_vector|k_csr_flat|k_dense_cluster"
for spec in "C1 3" "C2 3" "C3 3" "C4 3" "C5 4"; do
  set -- $spec
  extra=""; [ $1 = C5 ] && extra="--cg-iters 2"
  timeout 900 ncu --set full --clock-control none --import-source on -k "$KR" -s $2 -c 1 -o gpurun_out/prof_$1 python bench.py --config $1 --steps 1 --warmup 3 $extra --no-e2e --no-cpu-baseline > /dev/null 2>&1
  if [ -f gpurun_out/prof_$1.ncu-rep ]; then
    ncu -i gpurun_out/prof_$1.ncu-rep --page raw --csv > gpurun_out/prof_$1_raw.csv 2>/dev/null
    ncu -i gpurun_out/prof_$1.ncu-rep --page details > gpurun_out/prof_$1_details.txt 2>/dev/null
    rm -f gpurun_out/prof_$1.ncu-rep
  fi
done
du -sh gpurun_out

#!/bin/bash
# One GPU session: tests, benches, ncu evidence.  Outputs under gpurun_out/.
set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 -rf > gpurun_out/pytest_gpu.log 2>&1
tail -5 gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -c 400 gpurun_out/bench_default.json
for c in C1 C3 C4 C5; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
timeout 600 python bench.py --config C2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --force-dist > gpurun_out/bench_C2_dist.json 2> gpurun_out/bench_C2_dist.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in C2 C3 C4; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_$c.csv python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_dense_vector -s 3 -c 1 -o gpurun_out/prof_C2 python bench.py --config C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_csr -s 3 -c 1 -o gpurun_out/prof_C3 python bench.py --config C3 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_csr -s 3 -c 1 -o gpurun_out/prof_C4 python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_dense_vector -s 4 -c 1 -o gpurun_out/prof_C5 python bench.py --config C5 --steps 1 --warmup 3 --cg-iters 2 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_dense_vector -s 3 -c 1 -o gpurun_out/prof_C1 python bench.py --config C1 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
for c in C1 C2 C3 C4 C5; do
  if [ -f gpurun_out/prof_$c.ncu-rep ]; then
    ncu -i gpurun_out/prof_$c.ncu-rep --page raw --csv > gpurun_out/prof_${c}_raw.csv 2>/dev/null
    ncu -i gpurun_out/prof_$c.ncu-rep --page details > gpurun_out/prof_${c}_details.txt 2>/dev/null
    ncu -i gpurun_out/prof_$c.ncu-rep --page source --csv > gpurun_out/prof_${c}_source.csv 2>/dev/null
    rm -f gpurun_out/prof_$c.ncu-rep
  fi
done
du -sh gpurun_out; ls gpurun_out

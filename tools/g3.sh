set -u
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k "regex:k_csr" -c 1 -o gpurun_out/c3v11 \
  python bench.py --config C3 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --launch 11,4,4,0 > gpurun_out/c3v11_bench.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k "regex:k_csr_flat" -c 1 -o gpurun_out/c4 \
  python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/c4_bench.log 2>&1
for f in c3v11 c4; do
  ncu -i gpurun_out/$f.ncu-rep --page raw --csv > gpurun_out/${f}_raw.csv
  ncu -i gpurun_out/$f.ncu-rep --page details > gpurun_out/${f}_details.txt
  ncu -i gpurun_out/$f.ncu-rep --page source --csv --print-source sass > gpurun_out/${f}_sass.csv
  rm -f gpurun_out/$f.ncu-rep
done
ls -la gpurun_out

#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
CS=$(command -v compute-sanitizer || echo /usr/local/cuda/bin/compute-sanitizer)
echo "sanitizer: $CS"
for t in memcheck racecheck synccheck; do
  echo "## $t"; timeout 1500 $CS --tool $t python tools/sanitize.py > gpurun_out/r02c_san_$t.log 2>&1; echo "rc=$?"
  grep -E "COMPUTE-SANITIZER|ERROR SUMMARY|RACECHECK SUMMARY|sanitize driver" gpurun_out/r02c_san_$t.log | head; tail -3 gpurun_out/r02c_san_$t.log
done > gpurun_out/r02c_sanitizer.txt 2>&1
cat gpurun_out/r02c_sanitizer.txt

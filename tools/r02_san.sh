#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for t in memcheck racecheck synccheck; do
  echo "## $t"; timeout 1500 compute-sanitizer --tool $t python tools/sanitize.py 2>&1 | grep -E "COMPUTE-SANITIZER|ERROR SUMMARY|RACECHECK SUMMARY|SYNCCHECK|sanitize driver|Error|error" | head -20
done > gpurun_out/r02_sanitizer.txt
cat gpurun_out/r02_sanitizer.txt

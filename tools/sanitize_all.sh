#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_cases.py (run under gpurun)
mkdir -p gpurun_out/sanitizer
for t in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_cases.py > gpurun_out/sanitizer/$t.log 2>&1
  echo "$t rc=$?"; tail -3 gpurun_out/sanitizer/$t.log
done

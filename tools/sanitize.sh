#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py (run on the GPU box).
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|sanitize run ok" gpurun_out/sanitize_$tool.log | tail -2
done

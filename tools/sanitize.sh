#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py (run on the GPU box).
# initcheck does not track bulk-tensor (TMA) stores as initialising global
# memory, so it runs with the register-store epilogues (PARAPROX_TMA_STORE=0);
# memcheck / racecheck / synccheck run the default (TMA-store) kernels.
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  if [ $tool = initcheck ]; then export PARAPROX_TMA_STORE=0; fi
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|sanitize run ok" gpurun_out/sanitize_$tool.log | tail -2
done
unset PARAPROX_TMA_STORE

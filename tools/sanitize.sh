#!/bin/bash
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --target-processes all --print-limit 20 --error-exitcode 9 \
      python tools/sanitize_run.py > gpurun_out/${TAG:-r01b}_sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -4 gpurun_out/${TAG:-r01b}_sanitize_$tool.log
done

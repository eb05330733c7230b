#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck over scripts/sanitize_run.py
# (every class, both variants, all dtypes, scatter, host calls, device builder).  Logs to gpurun_out/.
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ $tool = memcheck ] && extra="--leak-check full"
  timeout 1800 compute-sanitizer --tool $tool $extra --target-processes all --print-limit 50 \
     python scripts/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|LEAK SUMMARY|sanitize workload ok" gpurun_out/sanitize_$tool.log | tail -3
done

#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small invocations of every primitive
set -x
for tool in memcheck racecheck synccheck; do
  compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_cases.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool exit=$?"
done

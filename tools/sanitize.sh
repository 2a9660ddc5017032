#!/bin/bash
# compute-sanitizer over the small scenarios (run under gpurun)
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  echo "=== $tool"
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_scenarios.py 2>&1 | tail -25
done > gpurun_out/sanitize.txt 2>&1

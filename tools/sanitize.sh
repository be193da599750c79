#!/bin/bash
# compute-sanitizer over tools/sanitize_probe.py (one tool per run; summaries in gpurun_out/)
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_probe.py \
      > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize_summary.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|Error|Hazard" gpurun_out/sanitize_$tool.log | tail -5 >> gpurun_out/sanitize_summary.txt
done

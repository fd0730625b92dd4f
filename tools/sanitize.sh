#!/bin/bash
# compute-sanitizer over the tiny windowed training; summaries -> gpurun_out/sanitize_*.txt
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=900
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
      python tools/sanitize_run.py > gpurun_out/sanitize_$tool.txt 2>&1
  echo "== $tool rc=$?"; grep -E "ERROR SUMMARY|SANITIZE_RUN_OK|RACECHECK SUMMARY" gpurun_out/sanitize_$tool.txt | tail -3
done

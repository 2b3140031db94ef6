#!/bin/bash
# compute-sanitizer over small runs of every variant/mode.  Usage: bash scripts/sanitize.sh TAG
TAG=${1:-san}; OUT=gpurun_out/$TAG; mkdir -p $OUT
for tool in memcheck synccheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --target-processes all \
    python scripts/sanitize_run.py > $OUT/$tool.txt 2>&1
  echo "$tool rc=$?" | tee -a $OUT/summary.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|SANITIZE_RUN_DONE|Error|Hazard" $OUT/$tool.txt | sort | uniq -c | head -8 | tee -a $OUT/summary.txt
done

#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize.py
cd "$(dirname "$0")/.."
OUT=${1:-gpurun_out/sanitizer.txt}
: > $OUT
for tool in memcheck racecheck synccheck; do
  echo "=== compute-sanitizer --tool $tool" >> $OUT
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py >> $OUT 2>&1
  echo "exit=$?" >> $OUT
done
grep -E "===|ERROR SUMMARY|RACECHECK SUMMARY|exit=|^ok" $OUT

#!/bin/bash
# TMA streaming characterisation: 1 producer thread, ring of S slots x chunk KB (~192 KB total)
cd "$(dirname "$0")/.."
bash tools/build_bench.sh >/dev/null 2>&1
B=tools/stream_bench
for spec in "2 96" "4 48" "8 24" "16 12" "32 6" "48 4" "16 4" "16 6" "32 4" "47 4"; do
  set -- $spec
  timeout 30 $B 1024 $1 $2 64 0 || echo "chunk $1 S $2 failed"
done
for L in 2 4 8; do timeout 30 $B 1024 32 6 $L 5 || echo "lanes $L failed"; done
timeout 30 $B 1024 16 8 1024 3 || echo "ldg failed"

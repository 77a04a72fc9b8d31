#!/bin/bash
# bulk-TMA streaming characterisation (1 producer thread per SM): chunk KB x slots. Each run bounded.
B=tools/stream_bench
for spec in "64 3" "32 6" "32 4" "32 3" "16 12" "16 8" "16 6" "16 4" "8 24" "8 12" "4 24"; do
  set -- $spec
  timeout 30 $B 1024 $1 $2 64 0 || echo "chunk $1 S $2 failed/timeout"
done
timeout 30 $B 1024 16 8 1024 3 || echo "ldg failed"

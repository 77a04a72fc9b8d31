#!/bin/bash
# stage-shape sweep for the tcgen05 kernel: G (GT columns per stage) x S (ring slots)
for spec in "4 4" "3 5" "3 6" "2 8" "2 6"; do
  set -- $spec
  rm -f gpurun_out/gs.json
  SPINFER_KERNEL=tc SPINFER_G=$1 SPINFER_S=$2 timeout 120 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --json-out gpurun_out/gs.json > /dev/null 2>&1
  python -c "import json;d=json.load(open('gpurun_out/gs.json'));print('G=$1 S=$2', round(d['us_per_spmm'],1), round(d['us_median'],1))" 2>/dev/null || echo "G=$1 S=$2 failed"
done

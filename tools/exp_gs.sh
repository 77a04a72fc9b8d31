#!/bin/bash
# production kernel, stage shape sweep (SPINFER_G / SPINFER_S caps)
for gs in ${@:-"5 3" "4 4" "4 3" "3 5"}; do set -- ${gs/_/ }
  SPINFER_G=$1 SPINFER_S=$2 timeout 120 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --json-out gpurun_out/gs_$1_$2.json > /dev/null 2>&1
  python -c "import json;d=json.load(open('gpurun_out/gs_$1_$2.json'));print('G=$1 S=$2 us',round(d['us_per_spmm'],1))"
done

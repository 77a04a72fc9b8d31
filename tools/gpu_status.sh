#!/bin/bash
# re-entry check: gpu tests, then mma vs tc bench A/B
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
for k in mma tc mma tc; do
  rm -f gpurun_out/s.json
  SPINFER_KERNEL=$k timeout 120 python bench.py --steps 30 --warmup 3 --no-cpu-baseline --no-e2e --json-out gpurun_out/s.json > /dev/null 2>gpurun_out/s_$k.err
  python -c "import json;d=json.load(open('gpurun_out/s.json'));print('$k', round(d['us_per_spmm'],1), round(d['us_median'],1), d.get('cublas_fp16',{}).get('us'))" || tail -3 gpurun_out/s_$k.err
done

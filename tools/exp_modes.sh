#!/bin/bash
# Timing experiments: SPINFER_DEBUG_MODE (bit0 consumers idle, bit1 scan idle) x stage shape (G, S).
mkdir -p gpurun_out
run() {  # tag, env...
  local tag=$1; shift
  env "$@" timeout 120 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --json-out gpurun_out/exp_$tag.json > gpurun_out/exp_$tag.log 2>&1
  python -c "import json;d=json.load(open('gpurun_out/exp_$tag.json'));print('$tag', ' '.join('$*'.split()), 'us',round(d['us_per_spmm'],1),'GB/s',round(d['value']))" 2>/dev/null || { echo "$tag FAILED"; tail -3 gpurun_out/exp_$tag.log; }
}
if [ "$1" = tests ]; then timeout 600 python -m pytest tests/test_spmm_gpu.py -x -q 2>&1 | tail -2; shift; fi
run m0 SPINFER_DEBUG_MODE=0
run m1 SPINFER_DEBUG_MODE=1
run m3 SPINFER_DEBUG_MODE=3
for gs in "$@"; do set -- $gs
  run m0_g$1s$2 SPINFER_DEBUG_MODE=0 SPINFER_G=$1 SPINFER_S=$2
  run m3_g$1s$2 SPINFER_DEBUG_MODE=3 SPINFER_G=$1 SPINFER_S=$2
done

#!/bin/bash
run() { local tag=$1; shift; export SPINFER_LIB=$PWD/paper_conf_eurosys_fanydlgww025_b200/libspinfer_instr.so
  env "$@" timeout 120 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --json-out gpurun_out/exp_$tag.json > gpurun_out/exp_$tag.log 2>&1
  python -c "import json;d=json.load(open('gpurun_out/exp_$tag.json'));print('$tag', ' '.join('$*'.split()), 'us',round(d['us_per_spmm'],1))" 2>/dev/null || { echo "$tag FAILED"; tail -3 gpurun_out/exp_$tag.log; }
}
if [ "$1" = tests ]; then timeout 600 python -m pytest tests/test_spmm_gpu.py -x -q 2>&1 | tail -2; shift; fi
for m in ${@:-0 3 4 5}; do run m$m SPINFER_DEBUG_MODE=$m; done

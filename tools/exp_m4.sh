#!/bin/bash
# instrumented build: full (m0) vs consumers-only (m4: reuse stage 0, no waits) vs consumers idle (m1)
L=$PWD/paper_conf_eurosys_fanydlgww025_b200/${LIBNAME:-libspinfer_dbg.so}
for m in ${MODES:-0 0 4 1 3 5}; do
  env SPINFER_LIB=$L SPINFER_DEBUG_MODE=$m timeout 120 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --json-out gpurun_out/fl.json > /dev/null 2>&1
  python -c "import json;d=json.load(open('gpurun_out/fl.json'));print('m$m', round(d['us_per_spmm'],1))"
done

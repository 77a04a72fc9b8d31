#!/bin/bash
# Debug-mode timing (libspinfer_dbg.so: SPINFER_DEBUG_MODE bits, no trace). MODES="0 4 ..." bash tools/exp_m4.sh
# bits: 1 consumers skip decode/MMA, 2 scan skips work, 4 consumers reuse stage 0 (no waits),
#       8 skip epilogue + fix-up, 16 consumers skip the stage loop
L=$PWD/paper_conf_eurosys_fanydlgww025_b200/${LIBNAME:-libspinfer_dbg.so}
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas > /dev/null 2>&1   # warm the box
for m in ${MODES:-0 4 1 5}; do
  rm -f gpurun_out/fl.json
  env SPINFER_LIB=$L SPINFER_DEBUG_MODE=$m timeout 180 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --json-out gpurun_out/fl.json > gpurun_out/fl_m$m.log 2>&1
  rc=$?
  python -c "import json;d=json.load(open('gpurun_out/fl.json'));print('m$m', round(d['us_per_spmm'],1))" 2>/dev/null || { echo "m$m FAILED rc=$rc"; tail -3 gpurun_out/fl_m$m.log; }
done

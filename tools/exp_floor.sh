#!/bin/bash
# Debug-mode floors with the instrumented build: mode 0 (full), 1 (consumers idle), 3 (consumers + scan idle)
L=$PWD/paper_conf_eurosys_fanydlgww025_b200/libspinfer_instr.so
for g in "$@"; do for m in 0 1 3; do
  env SPINFER_LIB=$L SPINFER_DEBUG_MODE=$m SPINFER_G=$g timeout 120 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --json-out gpurun_out/fl.json > /dev/null 2>&1
  python -c "import json;d=json.load(open('gpurun_out/fl.json'));print('G$g m$m', round(d['us_per_spmm'],1))"
done; done
SPINFER_LIB=$L SPINFER_G=4 SPINFER_TRACE=/tmp/tr.bin python tools/trace_run.py > gpurun_out/trace_g4.txt 2>&1
SPINFER_LIB=$L SPINFER_G=4 SPINFER_DEBUG_MODE=1 SPINFER_TRACE=/tmp/tr.bin python tools/trace_run.py > gpurun_out/trace_g4_m1.txt 2>&1

#!/bin/bash
# one gpurun call: spmm parity tests, then interleaved A/B timing of the current build vs libspinfer_prev.so
timeout 600 python -m pytest tests/test_spmm_gpu.py -x -q 2>&1 | tail -3
bash tools/ab.sh "prev:libspinfer_prev.so:" "cur:libspinfer.so:" "$@" 2>&1 | tee gpurun_out/ab_cur.txt

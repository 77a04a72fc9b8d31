#!/bin/bash
# stage timeline (instrumented build) + one ncu source-level capture of k_spmm; summaries to gpurun_out/
mkdir -p gpurun_out
timeout 300 python tools/trace_run.py > gpurun_out/trace.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 \
    -o gpurun_out/prof_diag python bench.py --profile --steps 2 --warmup 3 > gpurun_out/ncu_diag.log 2>&1
python tools/ncu_hot.py gpurun_out/prof_diag.ncu-rep 60 > gpurun_out/hot.txt 2>&1

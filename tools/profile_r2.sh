#!/bin/bash
# Round-2 profile captures (GPU box): ncu --set full of the three kernels on their headline shapes,
# the launch list of a short bench.py run, summaries in gpurun_out/.
cd "$(dirname "$0")/.."
set -x
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_dw -s 3 -c 1 -o gpurun_out/r2_dw \
  python bench.py --profile --steps 1 --warmup 3 > gpurun_out/r2_dw_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_tc -s 3 -c 1 -o gpurun_out/r2_tc32 \
  python bench.py --profile --steps 1 --warmup 3 --N 32 > gpurun_out/r2_tc32_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_wide -s 2 -c 1 -o gpurun_out/r2_wide4096 \
  python tools/wide_one.py 28672 8192 4096 > gpurun_out/r2_wide_ncu.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2_launches.csv \
  python bench.py --steps 5 --warmup 3 --no-extras --no-cpu-baseline > gpurun_out/r2_launch_bench.log 2>&1
for t in r2_dw r2_tc32 r2_wide4096; do
  python tools/ncu_summary.py gpurun_out/$t.ncu-rep > gpurun_out/${t}_summary.txt 2>&1
done

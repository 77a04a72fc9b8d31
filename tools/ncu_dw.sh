#!/bin/bash
# one ncu --set full capture of the SpMM kernel (development): ncu_dw.sh TAG [bench.py args...]
cd "$(dirname "$0")/.."
TAG=${1:-dw}; shift
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 \
  -o gpurun_out/$TAG python bench.py --profile --steps 1 --warmup 3 "$@" > gpurun_out/${TAG}_ncu.log 2>&1
python tools/ncu_summary.py gpurun_out/$TAG.ncu-rep > gpurun_out/${TAG}_summary.txt 2>&1
cat gpurun_out/${TAG}_summary.txt

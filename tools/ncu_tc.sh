#!/bin/bash
# ncu full capture of the SpMM kernel (config 2). Usage: ncu_tc.sh TAG [kernel-regex] (env passes through)
TAG=${1:-tc}; RX=${2:-k_spmm}
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$RX -s 3 -c 1 -o gpurun_out/prof_${TAG} python bench.py --profile --steps 2 --warmup 3 > gpurun_out/ncu_${TAG}.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_${TAG}.log

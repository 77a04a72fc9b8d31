#!/bin/bash
# tests + bench (tc and mma) + stage trace. Usage: gpu_tc2.sh TAG
TAG=${1:-tc}
bash tools/gpu_tc.sh $TAG
timeout 300 python tools/trace_tc.py > gpurun_out/trace_$TAG.txt 2>&1

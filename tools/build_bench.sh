#!/bin/bash
# Build the micro-benchmarks (experiment tools, not product): tools/<name> from tools/<name>.cu
cd "$(dirname "$0")"
for f in alu_bench alu_bench2 lds128_bench mio_bench smem_bench stream_bench launch_probe tc_probe; do
  [ -f $f.cu ] && nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o $f $f.cu
done

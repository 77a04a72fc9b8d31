#!/bin/bash
# One GPU iteration: [tests] bench [ncu full capture of the SpMM kernel]. Usage: gpu_iter.sh TAG [tests] [ncu]
TAG=${1:-it}; shift
mkdir -p gpurun_out
for a in "$@"; do
  if [ "$a" = tests ]; then
    timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_${TAG}.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_${TAG}.log
  fi
done
timeout 300 python bench.py --steps 30 --warmup 5 --json-out gpurun_out/bench_${TAG}.json > gpurun_out/bench_${TAG}.log 2>&1
for a in "$@"; do
  if [ "$a" = ncu ]; then
    timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv python bench.py --profile --steps 5 --warmup 3 > /dev/null 2>&1
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 -o gpurun_out/prof_${TAG} python bench.py --profile --steps 2 --warmup 3 > gpurun_out/ncu_${TAG}.log 2>&1
  fi
done
tail -3 gpurun_out/pytest_${TAG}.log 2>/dev/null; python - <<PY
import json
d=json.load(open("gpurun_out/bench_${TAG}.json"))
print("us", round(d["us_per_spmm"],2), "GB/s", round(d["value"],1), "frac", round(d["roofline"]["frac"],3), "cublas_us", d["cublas_fp16"] and round(d["cublas_fp16"]["us"],2), "clk", d["clocks"])
PY

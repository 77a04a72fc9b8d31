#!/bin/bash
# tcgen05 path bring-up: GPU tests (short timeout), then bench of both kernels. Usage: gpu_tc.sh TAG
TAG=${1:-tc}
mkdir -p gpurun_out
SPINFER_KERNEL=tc timeout 300 python -m pytest tests/test_spmm_gpu.py -x -q > gpurun_out/pytest_${TAG}.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_${TAG}.log
tail -15 gpurun_out/pytest_${TAG}.log
for k in tc mma; do  # SPINFER_KERNEL selects the kernel variant
  SPINFER_KERNEL=$k timeout 120 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e --json-out gpurun_out/bench_${TAG}_$k.json > gpurun_out/bench_${TAG}_$k.log 2>&1
  python -c "import json;d=json.load(open('gpurun_out/bench_${TAG}_$k.json'));print('$k', 'us', round(d['us_per_spmm'],2), 'med', round(d['us_median'],2), 'frac', round(d['roofline']['frac'],3), 'cublas', d['cublas_fp16'] and round(d['cublas_fp16']['us'],2))" || tail -5 gpurun_out/bench_${TAG}_$k.log
done

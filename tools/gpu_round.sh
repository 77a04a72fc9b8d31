#!/bin/bash
# Round deliverables in one gpurun call: full GPU tests, the default bench line (+ reference
# arm), the ncu launch list of the bench command, one ncu --set full capture of k_spmm.
# Usage (under gpurun): bash tools/gpu_round.sh TAG      -> gpurun_out/round_TAG/*
TAG=${1:-r1}
OUT=gpurun_out/round_$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > $OUT/gpu.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
timeout 600 python bench.py > $OUT/bench.jsonl 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/bench.err
timeout 600 python bench.py --impl reference > $OUT/bench_ref.jsonl 2> $OUT/bench_ref.err
# launch list of the bench command (cold-cache, serialised: compare shares, not absolutes)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $OUT/ncu_launch.log 2>&1
# one full capture of the hot kernel
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 \
    -o $OUT/prof_spmm python bench.py --profile --steps 2 --warmup 3 > $OUT/ncu_full.log 2>&1
ls -la $OUT

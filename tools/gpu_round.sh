#!/bin/bash
# Round deliverables in one gpurun call: the default bench line (+ N = 32 and the reference arm), the
# ncu launch list of the bench command, one ncu --set full capture of the N <= 16 kernel with its
# summary and hottest SASS. (GPU tests and smoke run separately.) Usage (under gpurun):
#   bash tools/gpu_round.sh TAG
cd "$(dirname "$0")/.."
TAG=${1:-r2c}
OUT=gpurun_out/round_$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > $OUT/gpu.txt 2>&1
timeout 900 python bench.py > $OUT/bench.jsonl 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/bench.err
timeout 600 python bench.py --N 32 --no-extras > $OUT/bench_n32.jsonl 2> $OUT/bench_n32.err
timeout 600 python bench.py --impl reference > $OUT/bench_ref.jsonl 2> $OUT/bench_ref.err
# launch list of the bench command (cold-cache, serialised: compare shares, not absolutes)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras > $OUT/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_dw -s 3 -c 1 \
    -o $OUT/prof_dw python bench.py --profile --steps 1 --warmup 3 > $OUT/ncu_full.log 2>&1
python tools/ncu_summary.py $OUT/prof_dw.ncu-rep > $OUT/ncu_summary.txt 2>&1
python tools/ncu_hot.py $OUT/prof_dw.ncu-rep 40 > $OUT/ncu_hot.txt 2>&1
ls -la $OUT

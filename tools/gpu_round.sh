#!/bin/bash
# Round deliverables in one gpurun call: full GPU tests, smoke, the default bench line (+ reference
# arm), the ncu launch list of the bench command, one ncu --set full capture of each kernel
# (k_spmm at N=16, k_spmm_tc at N=32) with summaries. Usage (under gpurun): bash tools/gpu_round.sh TAG
TAG=${1:-r1}
OUT=gpurun_out/round_$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > $OUT/gpu.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 300 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
timeout 600 python bench.py > $OUT/bench.jsonl 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/bench.err
timeout 600 python bench.py --N 32 > $OUT/bench_n32.jsonl 2> $OUT/bench_n32.err
timeout 600 python bench.py --impl reference > $OUT/bench_ref.jsonl 2> $OUT/bench_ref.err
# launch list of the bench command (cold-cache, serialised: compare shares, not absolutes)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $OUT/ncu_launch.log 2>&1
# one full capture of each hot kernel
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 \
    -o $OUT/prof_spmm python bench.py --profile --steps 2 --warmup 3 > $OUT/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_tc -s 3 -c 1 \
    -o $OUT/prof_spmm_tc32 python bench.py --profile --N 32 --steps 2 --warmup 3 > $OUT/ncu_full_tc.log 2>&1
python tools/ncu_summary.py $OUT/prof_spmm.ncu-rep > $OUT/ncu_summary.txt 2>&1
python tools/ncu_summary.py $OUT/prof_spmm_tc32.ncu-rep > $OUT/ncu_summary_tc32.txt 2>&1
python tools/ncu_hot.py $OUT/prof_spmm.ncu-rep 40 > $OUT/ncu_hot.txt 2>&1
ncu -i $OUT/prof_spmm.ncu-rep --page details --csv > $OUT/ncu_details.csv 2>&1
timeout 300 python tools/trace_run.py > $OUT/trace.txt 2>&1
ls -la $OUT

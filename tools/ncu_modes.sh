#!/bin/bash
for m in 0 3 4 5; do
  SPINFER_DEBUG_MODE=$m timeout 300 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,sm__cycles_active.avg --clock-control none -k regex:k_spmm -s 3 -c 1 --csv python bench.py --profile --steps 1 --warmup 3 2>/dev/null | grep -E "gpu__time|inst_executed|cycles_active" | awk -F'","' -v m=$m '{print "mode",m,$(NF-2),$NF}'
done
SPINFER_DEBUG_MODE=4 timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 -o gpurun_out/prof_m4 python bench.py --profile --steps 2 --warmup 3 > /dev/null 2>&1

#!/bin/bash
# A/B timing of library variants on the same box, interleaved: ab.sh "tag:lib:ENV=..." ...
# (extra bench.py arguments via $BENCH_ARGS, e.g. BENCH_ARGS='--N 32')
for rep in 1 2 3; do
  for spec in "$@"; do
    IFS=: read tag lib envs <<< "$spec"
    env SPINFER_LIB=$PWD/paper_conf_eurosys_fanydlgww025_b200/$lib $envs timeout 120 python bench.py $BENCH_ARGS --steps 30 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --no-extras --json-out gpurun_out/ab.json > /dev/null 2>&1
    python -c "import json;d=json.load(open('gpurun_out/ab.json'));print('$tag', round(d['us_per_spmm'],1))"
  done
done | sort | awk '{a[$1]=a[$1]" "$2} END {for (k in a) print k, a[k]}'

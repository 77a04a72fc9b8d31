timeout 900 python -m pytest tests -m gpu -x -q --timeout 120 2>&1 | tail -3
bash tools/ab.sh "base:libspinfer_base.so:" "cur:libspinfer_cur.so:"
for N in 8 32; do timeout 100 python bench.py --N $N --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --json-out gpurun_out/nn.json >/dev/null 2>&1 && python -c "import json;d=json.load(open('gpurun_out/nn.json'));print('N$N', round(d['us_per_spmm'],1), round(d['us_median'],1), d['cublas_fp16']['us'])"; rm -f gpurun_out/nn.json; done

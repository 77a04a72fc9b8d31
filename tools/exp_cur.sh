SPINFER_KERNEL=tc timeout 600 python -m pytest tests/test_spmm_gpu.py -x -q --timeout 120 2>&1 | tail -2
BENCH_ARGS="--N 32" bash tools/ab.sh "tcnowf:libspinfer_tcnowf.so:" "tcwf:libspinfer_tcwf.so:"
timeout 200 env SPINFER_KERNEL=tc python tools/cta_times.py 32

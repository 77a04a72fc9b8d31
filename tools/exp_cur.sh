timeout 600 python -m pytest tests/test_spmm_gpu.py -x -q --timeout 120 -k "not tc" 2>&1 | tail -2
bash tools/ab.sh "nobmbar:libspinfer_nobmbar.so:" "bmbar:libspinfer_bmbar.so:"
BENCH_ARGS="--N 8" bash tools/ab.sh "nobmbar8:libspinfer_nobmbar.so:" "bmbar8:libspinfer_bmbar.so:"

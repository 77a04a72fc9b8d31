timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 2>&1 | tail -3
BENCH_ARGS="--N 32" bash tools/ab.sh "base32:libspinfer_base.so:" "desc32:libspinfer_tcdesc.so:"

SPINFER_G0=1 timeout 600 python -m pytest tests/test_spmm_gpu.py -x -q --timeout 120 -k "not tc" 2>&1 | tail -2
bash tools/ab.sh "g04:libspinfer_g0.so:SPINFER_G0=4" "g01:libspinfer_g0.so:SPINFER_G0=1" "g02:libspinfer_g0.so:SPINFER_G0=2"

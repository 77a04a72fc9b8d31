timeout 900 python -m pytest tests/test_spmm_gpu.py -x -q --timeout 300 2>&1 | tail -2
bash tools/ab.sh "noepi:libspinfer_noepi.so:" "epi2:libspinfer_epi2.so:"

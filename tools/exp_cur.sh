SPINFER_LIB=$PWD/paper_conf_eurosys_fanydlgww025_b200/libspinfer_prodbo.so timeout 900 python -m pytest tests/test_spmm_gpu.py -x -q --timeout 120 2>&1 | tail -2
bash tools/ab.sh "nofixbo:libspinfer_nofixbo.so:" "fixbo:libspinfer_fixbo.so:" "prodbo:libspinfer_prodbo.so:" "prodbo1k:libspinfer_prodbo1k.so:"

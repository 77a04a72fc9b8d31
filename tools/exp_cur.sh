SPINFER_LIB=$PWD/paper_conf_eurosys_fanydlgww025_b200/libspinfer_relcnt.so timeout 900 python -m pytest tests/test_spmm_gpu.py -x -q --timeout 300 2>&1 | tail -2
bash tools/ab.sh "norelcnt:libspinfer_norelcnt.so:" "relcnt:libspinfer_relcnt.so:"

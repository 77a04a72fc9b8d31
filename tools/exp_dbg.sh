export SPINFER_LIB=$PWD/paper_conf_eurosys_fanydlgww025_b200/libspinfer_ep.so
timeout 200 python -m pytest tests/test_spmm_gpu.py -x -q --timeout 60 2>&1 | tail -25

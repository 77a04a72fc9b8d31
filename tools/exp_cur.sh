SPINFER_BONUS=4 SPINFER_LIB=$PWD/paper_conf_eurosys_fanydlgww025_b200/libspinfer_bonus.so timeout 600 python -m pytest tests/test_spmm_gpu.py -x -q --timeout 120 -k "not tc" 2>&1 | tail -2
bash tools/ab.sh "base:libspinfer_base.so:" "b0:libspinfer_bonus.so:SPINFER_BONUS=0" "b8:libspinfer_bonus.so:SPINFER_BONUS=8" "b4:libspinfer_bonus.so:SPINFER_BONUS=4"

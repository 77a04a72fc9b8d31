#!/bin/bash
# build a variant library: mkvar.sh TAG "-DFOO=1 -DBAR=2"  -> paper_conf_eurosys_fanydlgww025_b200/libspinfer_TAG.so
P=paper_conf_eurosys_fanydlgww025_b200
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
  -shared -cudart static -I include $2 $P/csrc/*.cu -o $P/libspinfer_$1.so

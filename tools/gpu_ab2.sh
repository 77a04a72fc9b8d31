#!/bin/bash
cd "$(dirname "$0")/.."
for v in r0p0 r0p1 r1p0 r1p1; do SPINFER_LIB=$PWD/paper_conf_eurosys_fanydlgww025_b200/libspinfer_$v.so timeout 60 python tools/dw_quick.py parity 2>&1 | tail -1; done
bash tools/ab.sh "r0p0:libspinfer_r0p0.so:" "r0p1:libspinfer_r0p1.so:" "r1p0:libspinfer_r1p0.so:" "r1p1:libspinfer_r1p1.so:"

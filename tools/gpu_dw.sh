#!/bin/bash
# development run: quick parity + timing of the new kernel, A/B vs the round-1 kernel
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python tools/dw_quick.py parity 2>&1 | tail -30
timeout 300 python tools/dw_quick.py time 2>&1 | tail -10
SPINFER_KERNEL=mma timeout 200 python tools/dw_quick.py time 2>&1 | tail -5

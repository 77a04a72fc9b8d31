#!/bin/bash
cd "$(dirname "$0")/.."
timeout 90 python tools/dw_quick.py parity 2>&1 | tail -4
timeout 120 python tools/dw_quick.py time 2>&1 | tail -5
timeout 90 python tools/dw_prof.py > gpurun_out/prof.txt 2>&1; head -16 gpurun_out/prof.txt

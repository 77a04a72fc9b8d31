#!/bin/bash
B=tools/stream_bench
$B 512 64 3 64 0; $B 512 16 6 64 0 2; $B 512 8 6 64 0 2; $B 512 8 12 64 0 2; $B 512 4 12 64 0 4
for L in 2 4 8 16; do $B 512 16 8 $L 5; $B 512 32 6 $L 5; done
for np in 1 2 4; do for c in 8 16 32; do $B 512 $c 6 $((32*np+32)) 4; done; done
$B 512 16 6 96 4 2; $B 512 16 3 96 4 2

#!/bin/bash
mkdir -p gpurun_out
ASTRA_PB_VERBOSE=1 ASTRA_PB_SPIN=20000000 timeout 200 python scratch/pb_debug.py lstm 3 64 2048 > gpurun_out/r2_pb21.log 2>&1
for sa in 2 3; do for kb in 1 2; do
ASTRA_PB_SA=$sa ASTRA_PB_KB=$kb ASTRA_PB_VERBOSE=1 timeout 200 python scratch/pb_debug.py lstm 3 64 2048 2>&1 | grep fits >> gpurun_out/r2_pb21.log
done; done

#!/bin/bash
mkdir -p gpurun_out
ASTRA_PB_VERBOSE=1 timeout 200 python scratch/pb_debug.py lstm 3 64 2048 > gpurun_out/r2_pb22.log 2>&1
ASTRA_PB_FORCE=1 ASTRA_PB_SPIN=20000000 timeout 200 python scratch/pb_debug.py lstm 3 64 2048 2>&1 | sort | uniq -c | sort -rn | head -30 >> gpurun_out/r2_pb22.log
echo "rc=$?" >> gpurun_out/r2_pb22.log

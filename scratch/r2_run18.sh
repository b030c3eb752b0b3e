#!/bin/bash
mkdir -p gpurun_out
ASTRA_PB_SPIN=20000000 timeout 120 python scratch/pb_debug.py lstm 1 64 2048 > gpurun_out/r2_pb18.log 2>&1; echo "rc=$?" >> gpurun_out/r2_pb18.log
ASTRA_PB_SPIN=20000000 timeout 120 python scratch/pb_debug.py lstm 2 64 2048 2>&1 | sort | uniq -c | sort -rn | head -40 >> gpurun_out/r2_pb18.log; echo "rc=$?" >> gpurun_out/r2_pb18.log

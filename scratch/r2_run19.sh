#!/bin/bash
mkdir -p gpurun_out
for T in 1 2 5; do
ASTRA_PB_SPIN=20000000 timeout 200 python -X faulthandler scratch/pb_debug.py lstm $T 64 2048 2>&1 | sort | uniq -c | sort -rn | head -30 >> gpurun_out/r2_pb20.log; echo "rc=$?" >> gpurun_out/r2_pb20.log
done
ASTRA_PB_SPIN=20000000 timeout 200 python -X faulthandler scratch/pb_debug.py milstm 5 37 2000 2>&1 | sort | uniq -c | sort -rn | head -30 >> gpurun_out/r2_pb20.log; echo "rc=$?" >> gpurun_out/r2_pb20.log

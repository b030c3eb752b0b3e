#!/bin/bash
mkdir -p gpurun_out
O=gpurun_out/r2_pb_sweep.jsonl
PB_VARIANT="bwd=0,bptt=128.1.1,bpw=1,fwd=3" timeout 120 python scratch/pb_sweep.py >> $O 2>&1
for cfg in "2 3 2 2 -1" "4 3 4 2 0" "4 4 4 2 0" "2 8 2 4 0" "4 3 2 2 8" "4 3 2 2 16" "8 2 4 2 0" "4 2 4 4 0"; do
  set -- $cfg
  ASTRA_PB_KA=$1 ASTRA_PB_SA=$2 ASTRA_PB_KB=$3 ASTRA_PB_SB=$4 ASTRA_PB_RES=$5 timeout 120 python scratch/pb_sweep.py >> $O 2>&1
done

#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace6.jsonl
for cfg in "ASTRA_SB_DBG_MMA=0" "ASTRA_SB_DBG_MMA=1" "ASTRA_SB_DBG_MMA=3"; do
  env ASTRA_SB_CS=1 $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace6.jsonl 2>>gpurun_out/sb_trace6.err
done
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv >> gpurun_out/sb_trace6.err

#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace8.jsonl
for cfg in "ASTRA_SB_DBG_MMA=-1" "ASTRA_SB_AROWS=128" "ASTRA_SB_DBG_MMA=-1 ASTRA_SB_RES=0 ASTRA_SB_SB=8"; do
  env ASTRA_SB_CS=1 $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace8.jsonl 2>>gpurun_out/sb_trace8.err
done

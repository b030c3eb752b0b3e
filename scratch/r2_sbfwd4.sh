#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace4.jsonl
for cfg in "ASTRA_SB_CS=1" "ASTRA_SB_CS=1 ASTRA_SB_SA=2" "ASTRA_SB_CS=1 ASTRA_SB_RES=32"; do
  env $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace4.jsonl 2>>gpurun_out/sb_trace4.err
done

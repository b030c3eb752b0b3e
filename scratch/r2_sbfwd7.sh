#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace7.jsonl
for cfg in "ASTRA_SB_DBG_STALE=0" "ASTRA_SB_DBG_STALE=1" "ASTRA_SB_DBG_STALE=1 ASTRA_SB_SA=2"; do
  env ASTRA_SB_CS=1 $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace7.jsonl 2>>gpurun_out/sb_trace7.err
done

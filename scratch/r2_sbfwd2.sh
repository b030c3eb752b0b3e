#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "small_batch_persistent" > gpurun_out/sb_test2.log 2>&1
echo "rc=$?" >> gpurun_out/sb_test2.log
for cfg in "" "ASTRA_SB_SA=12" "ASTRA_SB_SA=12 ASTRA_SB_RES=8 ASTRA_SB_SB=8" "ASTRA_SB_SA=10 ASTRA_SB_RES=0 ASTRA_SB_SB=14" "ASTRA_SB_SA=16 ASTRA_SB_RES=4 ASTRA_SB_SB=6"; do
  env $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace.jsonl 2>>gpurun_out/sb_trace.err
done

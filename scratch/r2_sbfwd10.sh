#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace10.jsonl
ASTRA_SB_2D=1 timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "small_batch_persistent" > gpurun_out/sb_test10.log 2>&1
for cfg in "ASTRA_SB_DBG_MMA=-1 ASTRA_SB_2D=1" "ASTRA_SB_2D=1" "ASTRA_SB_2D=1 ASTRA_SB_CS=1"; do
  env $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace10.jsonl 2>>gpurun_out/sb_trace10.err
done

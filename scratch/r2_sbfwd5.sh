#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace5.jsonl
timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "small_batch_persistent" > gpurun_out/sb_test5.log 2>&1
ASTRA_SB_NR=8 timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "small_batch_persistent" >> gpurun_out/sb_test5.log 2>&1
echo "rc=$?" >> gpurun_out/sb_test5.log
for cfg in "ASTRA_SB_CS=1 ASTRA_SB_NR=0" "ASTRA_SB_CS=1 ASTRA_SB_NR=2" "ASTRA_SB_CS=1 ASTRA_SB_NR=4" "ASTRA_SB_CS=1 ASTRA_SB_NR=8" "ASTRA_SB_CS=4 ASTRA_SB_NR=8"; do
  env $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace5.jsonl 2>>gpurun_out/sb_trace5.err
done

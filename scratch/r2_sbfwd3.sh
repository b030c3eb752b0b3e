#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace3.jsonl
timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "small_batch_persistent or gate_chunking" > gpurun_out/sb_test3.log 2>&1
echo "rc=$?" >> gpurun_out/sb_test3.log
for cfg in "ASTRA_SB_CS=1" "ASTRA_SB_CS=2" "ASTRA_SB_CS=4" "ASTRA_SB_CS=4 ASTRA_SB_SA=16" "ASTRA_SB_CS=8" ; do
  env $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace3.jsonl 2>>gpurun_out/sb_trace3.err
done

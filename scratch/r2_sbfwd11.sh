#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace11.jsonl
timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "small_batch_persistent" > gpurun_out/sb_test11.log 2>&1
echo "rc=$?" >> gpurun_out/sb_test11.log
for cfg in "ASTRA_SB_KA=4" "ASTRA_SB_KA=8 ASTRA_SB_SA=2" "ASTRA_SB_KA=4 ASTRA_SB_SA=2 ASTRA_SB_KB=4" "ASTRA_SB_KA=2 ASTRA_SB_SA=4"; do
  env $cfg timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace11.jsonl 2>>gpurun_out/sb_trace11.err
done

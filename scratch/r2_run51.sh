#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_fullsize.py -q -x -k "attn or cfg4" > gpurun_out/r2_t51.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t51.log
for i in 1 2; do timeout 600 python scratch/cfg_bench.py cfg4 >> gpurun_out/r2_cfg51.jsonl 2>&1; done

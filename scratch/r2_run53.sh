#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_fullsize.py -q -x -k "attn or cfg4" > gpurun_out/r2_t53.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t53.log
for i in 1 2; do timeout 600 python scratch/cfg_bench.py cfg4 >> gpurun_out/r2_cfg53.jsonl 2>&1; done
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_acc --csv --log-file gpurun_out/r2_attnacc53.csv python scratch/prof_cfg4.py > /dev/null 2>&1

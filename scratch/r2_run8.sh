#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -q -x -k "scrn" > gpurun_out/r2_t8.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t8.log
timeout 900 python scratch/cfg_bench.py cfg2 > gpurun_out/r2_cfg2b.log 2>&1

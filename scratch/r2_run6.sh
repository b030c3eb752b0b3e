#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py -q -x -k "scrn" > gpurun_out/r2_t6.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t6.log
timeout 900 python scratch/cfg_bench.py cfg2 > gpurun_out/r2_cfg2.log 2>&1

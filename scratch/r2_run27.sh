#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py tests/test_gpu_trajectory.py -q -x > gpurun_out/r2_t27.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t27.log
timeout 300 python bench.py --steps 20 > gpurun_out/r2_b27_512.log 2>&1
timeout 300 python bench.py --steps 20 --batch 64 > gpurun_out/r2_b27_64.log 2>&1

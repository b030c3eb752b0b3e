#!/bin/bash
# round-2 baseline on one B200: GPU suite, bench at cfg5 and at B=64, the other configs
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2b_smi.txt
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2b_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2b_pytest.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r2b_bench512.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --batch 64 --no-cpu-baseline > gpurun_out/r2b_bench64.log 2>&1
timeout 900 python scratch/cfg_bench.py all > gpurun_out/r2b_cfgs.log 2>&1

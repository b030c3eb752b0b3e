#!/bin/bash
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2_pytest7.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_pytest7.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r2_bench7.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 --batch 64 --no-cpu-baseline > gpurun_out/r2_bench7_b64.log 2>&1
timeout 900 python scratch/cfg_bench.py all > gpurun_out/r2_cfgs7.log 2>&1

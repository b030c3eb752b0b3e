#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/ -m gpu -q -x > gpurun_out/r2_t38.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t38.log
timeout 300 python bench.py --steps 20 --batch 64 > gpurun_out/r2_b38_64.log 2>&1
timeout 300 python bench.py --steps 20 > gpurun_out/r2_b38_512.log 2>&1
timeout 900 python scratch/cfg_bench.py all > gpurun_out/r2_cfg38.jsonl 2>&1

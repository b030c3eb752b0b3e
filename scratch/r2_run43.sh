#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/ -m gpu -q -x > gpurun_out/r2_t43.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t43.log
timeout 600 python bench.py > gpurun_out/r2_b43.log 2>&1
timeout 900 python scratch/cfg_bench.py all > gpurun_out/r2_cfg43.jsonl 2>&1
timeout 400 python scratch/gemm_sweep2.py > gpurun_out/r2_gemm_sweep43.jsonl 2>&1

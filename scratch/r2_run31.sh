#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_gemm.py -q -x > gpurun_out/r2_t31.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t31.log
timeout 400 python scratch/gemm_sweep2.py > gpurun_out/r2_gemm_sweep31.jsonl 2>&1
ASTRA_GEMM_KB=1 timeout 400 python scratch/gemm_sweep2.py > gpurun_out/r2_gemm_sweep31_kb1.jsonl 2>&1

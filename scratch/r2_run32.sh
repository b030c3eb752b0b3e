#!/bin/bash
mkdir -p gpurun_out
timeout 400 python scratch/gemm_sweep2.py > gpurun_out/r2_gemm_sweep32.jsonl 2>&1
ASTRA_GEMM_KB=1 timeout 400 python scratch/gemm_sweep2.py > gpurun_out/r2_gemm_sweep32_kb1.jsonl 2>&1

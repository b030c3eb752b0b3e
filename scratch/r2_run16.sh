#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_lm.py -q -x -k "stream_schedules or embedding" > gpurun_out/r2_t16.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t16.log
timeout 600 python scratch/gemm_sweep.py > gpurun_out/r2_gemm_sweep16.jsonl 2>&1
timeout 600 python scratch/cfg_bench.py cfg2 > gpurun_out/r2_cfg16.jsonl 2>&1

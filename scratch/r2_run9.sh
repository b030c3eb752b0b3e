#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -q -x -k "rhn" > gpurun_out/r2_t9.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t9.log
timeout 900 python scratch/cfg_bench.py cfg3 > gpurun_out/r2_cfg3.log 2>&1

#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -q -x -k "rhn" > gpurun_out/r2_t11.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t11.log
timeout 300 python scratch/trace_rhn.py > gpurun_out/r2_trace_rhn2.log 2>&1
timeout 900 python scratch/cfg_bench.py cfg3 > gpurun_out/r2_cfg3b.log 2>&1

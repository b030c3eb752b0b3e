#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -q -x -k "rhn" > gpurun_out/r2_t57.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t57.log
timeout 900 compute-sanitizer --tool memcheck python scratch/sanitize_cases.py rhn_bptt > gpurun_out/r2_san57_mem.log 2>&1; echo "rc=$?" >> gpurun_out/r2_san57_mem.log
timeout 900 compute-sanitizer --tool synccheck python scratch/sanitize_cases.py rhn_bptt > gpurun_out/r2_san57_sync.log 2>&1; echo "rc=$?" >> gpurun_out/r2_san57_sync.log

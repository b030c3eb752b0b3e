#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_lm.py tests/test_gpu_cell.py -m gpu -q -k "never_blocks or fork_explores or tune" > gpurun_out/r3l_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3l_pytest.log
ASTRA_DUMP_REPORT=gpurun_out/r3l_report.json python bench.py --no-cpu-baseline > gpurun_out/r3l_bench.log 2>&1
python bench.py --no-cpu-baseline > gpurun_out/r3l_bench2.log 2>&1

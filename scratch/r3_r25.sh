#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3r25_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3r25_pytest.log
for r in 1 2; do timeout 300 python scratch/cfg_bench.py cfg4 >> gpurun_out/r3r25_cfg4.log 2>&1; done

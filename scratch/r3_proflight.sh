#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r3pl_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3pl_pytest.log
python bench.py --no-cpu-baseline > gpurun_out/r3pl_bench.log 2>&1
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r3pl_bench_b64.log 2>&1

#!/bin/bash
# Re-entry validation: full GPU suite, bench lines at B=512 and B=64, the other configs.
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/r3v_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3v_pytest.log
python bench.py > gpurun_out/r3v_bench.log 2>&1
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r3v_bench_b64.log 2>&1
timeout 900 python scratch/cfg_bench.py > gpurun_out/r3v_cfgs.log 2>&1

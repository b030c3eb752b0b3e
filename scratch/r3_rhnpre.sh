#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "rhn or scrn or trajectory or fullsize" > gpurun_out/r3rp_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3rp_pytest.log
for r in 1 2; do timeout 300 python scratch/cfg_bench.py cfg3 >> gpurun_out/r3rp_cfg3.log 2>&1; done
timeout 300 python scratch/cfg_bench.py cfg2 >> gpurun_out/r3rp_cfg2.log 2>&1

#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2s9_pytest_all.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2s9_pytest_all.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s9_smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/r2s9_smoke.txt
python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2s9_bench.log 2>&1

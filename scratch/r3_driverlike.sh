#!/bin/bash
# Driver-like sequence on the shipped build: GPU suite, smoke, default bench, reference arm.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2s8_driverlike_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2s8_driverlike_pytest.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s8_driverlike_smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/r2s8_driverlike_smoke.txt
python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2s8_driverlike_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/r2s8_driverlike_bench.log
timeout 600 python bench.py --impl reference --gpus 1 --steps 2 --warmup 1 > gpurun_out/r2s8_driverlike_ref.log 2>&1; echo "ref rc=$?" >> gpurun_out/r2s8_driverlike_ref.log
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r2s8_driverlike_bench_b64.log 2>&1
timeout 900 python scratch/cfg_bench.py > gpurun_out/r2s8_driverlike_cfgs.jsonl 2>&1

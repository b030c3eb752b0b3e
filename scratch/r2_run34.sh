#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/ -m gpu -q -x -k "rhn" > gpurun_out/r2_t34.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t34.log
timeout 600 python scratch/cfg_bench.py cfg3 > gpurun_out/r2_cfg34.jsonl 2>&1
ASTRA_RHN_KA=1 timeout 600 python scratch/cfg_bench.py cfg3 >> gpurun_out/r2_cfg34.jsonl 2>&1

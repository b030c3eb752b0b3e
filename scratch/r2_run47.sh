#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -m gpu -q -x -k "rhn or scrn" > gpurun_out/r2_t47.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t47.log
for i in 1 2; do timeout 600 python scratch/cfg_bench.py cfg3 >> gpurun_out/r2_cfg47.jsonl 2>&1; done

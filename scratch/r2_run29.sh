#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/ -m gpu -q -x -k "rhn" > gpurun_out/r2_t29.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t29.log
timeout 600 python scratch/cfg_bench.py cfg3 > gpurun_out/r2_cfg29.jsonl 2>&1

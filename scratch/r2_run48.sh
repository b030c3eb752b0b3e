#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -m gpu -q -x -k "rhn" > gpurun_out/r2_t48.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t48.log
timeout 300 python scratch/trace_rhn.py > gpurun_out/r2_trace_rhn16.log 2>&1
for i in 1 2; do timeout 600 python scratch/cfg_bench.py cfg3 >> gpurun_out/r2_cfg48.jsonl 2>&1; done

#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/ -m gpu -q -x -k "rhn" > gpurun_out/r2_t41.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t41.log
timeout 300 python scratch/trace_rhn.py > gpurun_out/r2_trace_rhn_tl.log 2>&1
timeout 600 python scratch/cfg_bench.py cfg3 > gpurun_out/r2_cfg41.jsonl 2>&1

#!/bin/bash
mkdir -p gpurun_out
ASTRA_DUMP_REPORT=gpurun_out/r3d_report.json python bench.py --no-cpu-baseline --steps 10 > gpurun_out/r3d_bench.log 2>&1

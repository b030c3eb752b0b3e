#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/ -m gpu -q -x -k "rhn" > gpurun_out/r2_t36.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t36.log
timeout 300 python scratch/trace_rhn.py > gpurun_out/r2_trace_rhn_c1.log 2>&1
ASTRA_RHN_KA=1 timeout 300 python scratch/trace_rhn.py > gpurun_out/r2_trace_rhn_c1_ka1.log 2>&1

#!/bin/bash
mkdir -p gpurun_out
timeout 300 python scratch/trace_rhn.py > gpurun_out/r2_trace_rhn_ka4.log 2>&1
ASTRA_RHN_KA=1 timeout 300 python scratch/trace_rhn.py > gpurun_out/r2_trace_rhn_ka1.log 2>&1
ASTRA_RHN_KA=13 timeout 300 python scratch/trace_rhn.py > gpurun_out/r2_trace_rhn_ka13.log 2>&1

#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/sb_trace12.jsonl
timeout 300 python scratch/trace_sbfwd.py >> gpurun_out/sb_trace12.jsonl 2>>gpurun_out/sb_trace12.err
